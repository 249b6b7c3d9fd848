# final: whole GPU suite, smoke, bench (driver flags), reference arm
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tests_r2fin.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_r2fin.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r2fin.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke_r2fin.log
timeout 900 python bench.py --steps 200 --warmup 5 > gpurun_out/bench_r2fin.json 2> gpurun_out/bench_r2fin.err; echo "bench rc=$?"
timeout 900 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/bench_ref_r2fin.json 2> gpurun_out/bench_ref_r2fin.err; echo "ref rc=$?"
python -c "
import json; d=json.load(open('gpurun_out/bench_r2fin.json')); print(d['value'], d['ms_per_step'], d['roofline']['frac'], json.dumps(d['e2e'])[:300]); print(d['workloads']['C4']['plans']['b200']['ms_per_step'])"

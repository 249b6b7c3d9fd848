# pdl=2 default: whole GPU suite, smoke, bench (driver flags), reference arm
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tests_r2pdl.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_r2pdl.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r2pdl.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke_r2pdl.log
timeout 900 python bench.py --steps 200 --warmup 5 > gpurun_out/bench_r2pdl.json 2> gpurun_out/bench_r2pdl.err; echo "bench rc=$?"
timeout 900 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/bench_ref_r2pdl.json 2> gpurun_out/bench_ref_r2pdl.err; echo "ref rc=$?"
python -c "
import json; d=json.load(open('gpurun_out/bench_r2pdl.json')); print(d['value'], d['ms_per_step'], d['roofline']['frac'], json.dumps(d['e2e'])[:300]); print(d['workloads']['C4']['plans']['b200']['ms_per_step'])"
timeout 300 python tools/sweep.py --config C4 --reps 5 '' 'pdl=0' 'pdl=1' '' > gpurun_out/r02_sweep_pdl_c4.jsonl 2>&1; cat gpurun_out/r02_sweep_pdl_c4.jsonl

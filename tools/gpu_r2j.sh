# r2j: final build -- whole GPU suite, smoke, bench N=1, reference arm
mkdir -p gpurun_out
KF_PARITY_LOG=gpurun_out/parity_r2j.jsonl timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tests_r2j.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_r2j.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r2j.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke_r2j.log
timeout 900 python bench.py --steps 200 --warmup 5 > gpurun_out/bench_r2j.json 2> gpurun_out/bench_r2j.err; echo "bench rc=$?"; head -c 300 gpurun_out/bench_r2j.json
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/bench_ref_r2j.json 2>&1; echo "ref rc=$?"

# r2v: geometry memo -- whole GPU suite, host-overhead probe, e2e probe, bench
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tests_r2v.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/tests_r2v.log
python tools/host_overhead_probe.py
timeout 600 python tools/e2e_probe.py C3 ''
timeout 900 python bench.py --steps 200 --warmup 5 > gpurun_out/bench_r2v.json 2> gpurun_out/bench_r2v.err; echo "bench rc=$?"; head -c 250 gpurun_out/bench_r2v.json

# kf_run_host_async: GPU tests, then the bench e2e
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "run_host" > gpurun_out/tests_r2as.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_r2as.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_r2as.json 2> gpurun_out/bench_r2as.err; echo "bench rc=$?"
python -c "
import json; d=json.load(open('gpurun_out/bench_r2as.json')); print(json.dumps(d['e2e'])); print(d['value'])"

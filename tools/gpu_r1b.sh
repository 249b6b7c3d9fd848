mkdir -p gpurun_out
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/tests_gpu.log 2>&1; echo "tests rc=$?"; tail -5 gpurun_out/tests_gpu.log
python tools/sweep.py --steps 100 --config C4 "" "KFUSE_SWAR=0" > gpurun_out/sweep_c4.jsonl 2>&1
for pl in unfused paper; do python tools/sweep.py --steps 100 --config C4 --plan $pl ""; done >> gpurun_out/sweep_c4.jsonl 2>&1
cat gpurun_out/sweep_c4.jsonl
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"; cat gpurun_out/bench.json

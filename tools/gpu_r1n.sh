mkdir -p gpurun_out
timeout 900 python tools/sweep.py --config C4 --plan b200 '' > gpurun_out/sweep_c4b.jsonl 2>&1; cat gpurun_out/sweep_c4b.jsonl
timeout 1800 python -m pytest tests -x -q -m gpu > gpurun_out/tests_gpu.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_gpu.log

mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu -k "swar or overlapped or run_host or full_size" > gpurun_out/tests_gpu_new.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_gpu_new.log
python tools/sweep.py --steps 100 --config enhance:2048:2048 "" "KFUSE_CODE_BUDGET=1000" "KFUSE_CODE_BUDGET=4000" > gpurun_out/sweep_enh.jsonl 2>&1; cat gpurun_out/sweep_enh.jsonl
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"; cut -c1-1500 gpurun_out/bench.json

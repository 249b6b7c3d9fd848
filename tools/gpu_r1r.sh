mkdir -p gpurun_out
timeout 900 python tools/sweep.py --config C4 --plan b200 '' 'KFUSE_ROLLED_EDGE_V=0' > gpurun_out/sweep_ev.jsonl 2>&1
timeout 600 python tools/sweep.py --config enhance:2048:2048 --plan b200 '' 'KFUSE_ROLLED_EDGE_V=0' >> gpurun_out/sweep_ev.jsonl 2>&1
cat gpurun_out/sweep_ev.jsonl
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/tests_gpu.log 2>&1; echo "tests rc=$?"; tail -5 gpurun_out/tests_gpu.log

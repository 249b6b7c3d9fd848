mkdir -p gpurun_out
timeout 1200 python tools/sweep.py --config copy:2048:2048 --plan b200 '' 'KFUSE_PERSIST=0' 'KFUSE_PERSIST_WAVES=2' > gpurun_out/sweep_p.jsonl 2>&1
timeout 1200 python tools/sweep.py --config C2 --plan b200 '' 'KFUSE_PERSIST=0' 'KFUSE_PERSIST_WAVES=2' >> gpurun_out/sweep_p.jsonl 2>&1
timeout 1200 python tools/sweep.py --config C3 --plan b200 '' 'KFUSE_PERSIST=0' 'KFUSE_PERSIST_WAVES=2' >> gpurun_out/sweep_p.jsonl 2>&1
timeout 1200 python tools/sweep.py --config C4 --plan b200 '' 'KFUSE_PERSIST=0' >> gpurun_out/sweep_p.jsonl 2>&1
timeout 1200 python tools/sweep.py --config C3 --plan unfused '' 'KFUSE_PERSIST=0' >> gpurun_out/sweep_p.jsonl 2>&1
cat gpurun_out/sweep_p.jsonl
timeout 900 python -m pytest tests -x -q -m gpu -k "strip_geometry or run_host or bands or workloads or tiny or random or modes" > gpurun_out/tests_gpu.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_gpu.log

mkdir -p gpurun_out
timeout 1200 python tools/sweep.py --config C3 --plan b200 '' 'KFUSE_QPTR=0' 'KFUSE_CONST_W=0' 'KFUSE_QPTR=0 KFUSE_CONST_W=0' > gpurun_out/sweep_q.jsonl 2>&1
timeout 600 python tools/sweep.py --config C3s --plan b200 '' 'KFUSE_QPTR=0 KFUSE_CONST_W=0' >> gpurun_out/sweep_q.jsonl 2>&1
timeout 600 python tools/sweep.py --config C2 --plan b200 '' 'KFUSE_QPTR=0 KFUSE_CONST_W=0' >> gpurun_out/sweep_q.jsonl 2>&1
timeout 600 python tools/sweep.py --config C4 --plan b200 '' 'KFUSE_QPTR=0 KFUSE_CONST_W=0' >> gpurun_out/sweep_q.jsonl 2>&1
cat gpurun_out/sweep_q.jsonl
timeout 900 python -m pytest tests -x -q -m gpu -k "strip_geometry or run_host or bands or workloads or tiny or random" > gpurun_out/tests_gpu.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_gpu.log

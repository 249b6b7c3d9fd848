mkdir -p gpurun_out
timeout 1200 python tools/sweep.py --config C3 --plan b200 '' 'KFUSE_V8=1' 'KFUSE_V8=1 KFUSE_SMEM_ROWS=8' 'KFUSE_V8=1 KFUSE_MINCTAS=16' > gpurun_out/sweep_v8.jsonl 2>&1
timeout 900 python tools/sweep.py --config C3s --plan b200 '' 'KFUSE_V8=1' >> gpurun_out/sweep_v8.jsonl 2>&1
timeout 900 python tools/sweep.py --config C2 --plan b200 '' 'KFUSE_V8=1' >> gpurun_out/sweep_v8.jsonl 2>&1
timeout 900 python tools/sweep.py --config copy:4096:4096 --plan b200 '' 'KFUSE_V8=1' >> gpurun_out/sweep_v8.jsonl 2>&1
cat gpurun_out/sweep_v8.jsonl
KFUSE_V8=1 timeout 1500 python -m pytest tests -x -q -m gpu -k "strip_geometry or run_host or bands or workloads or tiny or random or modes or fig4" > gpurun_out/tests_v8.log 2>&1; echo "tests v8 rc=$?"; tail -3 gpurun_out/tests_v8.log

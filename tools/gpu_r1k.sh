mkdir -p gpurun_out
timeout 1200 python tools/sweep.py --config C3 --plan b200 '' 'KFUSE_HEAVY_FIRST=0' 'KFUSE_MINCTAS=24' 'KFUSE_MINCTAS=20' 'KFUSE_NSTRIPS=118' 'KFUSE_NSTRIPS=148' 'KFUSE_NSTRIPS=169' 'KFUSE_NSTRIPS=200' 'KFUSE_NSTRIPS=236' 'KFUSE_NSTRIPS=296' 'KFUSE_MINCTAS=24 KFUSE_NSTRIPS=236' 'KFUSE_MINCTAS=24 KFUSE_NSTRIPS=200' > gpurun_out/sweep_geo.jsonl 2>&1; cat gpurun_out/sweep_geo.jsonl
timeout 900 python -m pytest tests -x -q -m gpu -k "strip_geometry or run_host or bands or workloads or tiny" > gpurun_out/tests_gpu.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_gpu.log

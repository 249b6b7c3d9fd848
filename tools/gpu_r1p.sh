mkdir -p gpurun_out
timeout 1200 python tools/sweep.py --config C3 --plan b200 '' 'KFUSE_CODE_BUDGET=1000' 'KFUSE_SMEM_ROWS=9' 'KFUSE_SMEM_ROWS=6' 'KFUSE_PREFETCH=2' '' > gpurun_out/sweep_r.jsonl 2>&1
cat gpurun_out/sweep_r.jsonl

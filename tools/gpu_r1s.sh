mkdir -p gpurun_out
timeout 1500 python tools/sweep.py --config C4 --plan b200 '' 'KFUSE_NSTRIPS=24' 'KFUSE_NSTRIPS=34' 'KFUSE_NSTRIPS=45' 'KFUSE_NSTRIPS=90' 'KFUSE_SWRING_CAP=100' 'KFUSE_SWRING_CAP=48' 'KFUSE_SMEM_ROWS=16' > gpurun_out/sweep_c4s.jsonl 2>&1
cat gpurun_out/sweep_c4s.jsonl

mkdir -p gpurun_out
timeout 1500 python tools/sweep.py --config C4 --plan b200 '' 'KFUSE_CODE_BUDGET=100000000' 'KFUSE_MINCTAS=8' 'KFUSE_MINCTAS=16' > gpurun_out/sweep_c4.jsonl 2>&1; cat gpurun_out/sweep_c4.jsonl

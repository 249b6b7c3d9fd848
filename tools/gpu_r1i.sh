mkdir -p gpurun_out
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/sq tools/ubench/sqrt_approx.cu && /tmp/sq
timeout 900 python tools/sweep.py --config C3 --plan b200 '' 'KFUSE_LDS_PF=0' 'KFUSE_PRO_RP=0' 'KFUSE_LDS_PF=0 KFUSE_PRO_RP=0' 'KFUSE_SMEM_ROWS=9' 'KFUSE_SMEM_ROWS=15' 'KFUSE_NSTRIPS=300' > gpurun_out/sweep_pf.jsonl 2>&1; cat gpurun_out/sweep_pf.jsonl
timeout 600 python tools/sweep.py --config C3s --plan b200 '' 'KFUSE_LDS_PF=0' > gpurun_out/sweep_pf2.jsonl 2>&1; cat gpurun_out/sweep_pf2.jsonl
timeout 600 python tools/sweep.py --config C4 --plan b200 '' 'KFUSE_LDS_PF=0' >> gpurun_out/sweep_pf2.jsonl 2>&1; tail -2 gpurun_out/sweep_pf2.jsonl
timeout 600 python tools/sweep.py --config C2 --plan b200 '' 'KFUSE_LDS_PF=0' >> gpurun_out/sweep_pf2.jsonl 2>&1; tail -2 gpurun_out/sweep_pf2.jsonl
timeout 1500 python -m pytest tests -x -q -m gpu -k "strip_geometry or run_host or bands or workloads or fig4 or tiny" > gpurun_out/tests_gpu.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_gpu.log

mkdir -p gpurun_out
timeout 900 python tools/sweep.py --config copy:2048:2048 --plan b200 '' > gpurun_out/sweep_c2.jsonl 2>&1
timeout 900 python tools/sweep.py --config blur:2048:2048 --plan b200 '' >> gpurun_out/sweep_c2.jsonl 2>&1
timeout 900 python tools/sweep.py --config C2 --plan b200 '' 'KFUSE_NSTRIPS=16' 'KFUSE_NSTRIPS=32' 'KFUSE_NSTRIPS=64' 'KFUSE_NSTRIPS=128' 'KFUSE_NSTRIPS=256' 'KFUSE_SMEM_ROWS=6' 'KFUSE_SMEM_ROWS=9' >> gpurun_out/sweep_c2.jsonl 2>&1
cat gpurun_out/sweep_c2.jsonl
for cfg in C2 C3s C4; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:kf_b -s 2 -c 1 -f -o gpurun_out/prof_${cfg} \
     python tools/prof_run.py --config $cfg --plan b200 > gpurun_out/ncu_${cfg}.log 2>&1; echo "ncu $cfg rc=$?"
done

# thread-block cluster launch experiment (CTA dispatch): C3, copy, C2, C4
for cfg in C3 copy:4096:4096 C2 C4; do
  timeout 300 python tools/sweep.py --config $cfg --lib testhooks --reps 7 '' 'cluster=2' 'cluster=4' 'cluster=8' ''
done > gpurun_out/r02_sweep_cluster.jsonl 2>&1
cat gpurun_out/r02_sweep_cluster.jsonl

# warm_skip 0 / 1 (guards in the loop) / 2 (own warm-up loop) A/B
for cfg in C4 enhance:2048:2048; do
  timeout 400 python tools/sweep.py --config $cfg --reps 7 '' 'warm_skip=2' 'warm_skip=0' '' 'warm_skip=2' 'warm_skip=0'
done > gpurun_out/r02_sweep_warm_skip2.jsonl 2>&1
cat gpurun_out/r02_sweep_warm_skip2.jsonl

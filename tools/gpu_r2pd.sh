for cfg in C1 C5 copy:4096:4096 sobel:2048:2048 enhance:2048:2048 C2 C3; do
  timeout 300 python tools/sweep.py --config $cfg --reps 7 '' 'pdl=1' '' 'pdl=1'
done > gpurun_out/r02_sweep_pdl_final.jsonl 2>&1
for cfg in C3 C2 C4; do
  timeout 300 python tools/sweep.py --config $cfg --plan unfused --reps 5 '' 'pdl=1' '' 'pdl=1'
done >> gpurun_out/r02_sweep_pdl_final.jsonl 2>&1
cat gpurun_out/r02_sweep_pdl_final.jsonl

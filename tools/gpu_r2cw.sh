for cfg in C3 C2 C4 C3s; do
  timeout 300 python tools/sweep.py --config $cfg --reps 7 '' 'cta_warps=2' 'cta_warps=4' 'pdl=1' ''
done > gpurun_out/r02_sweep_cta_warps_final.jsonl 2>&1
cat gpurun_out/r02_sweep_cta_warps_final.jsonl

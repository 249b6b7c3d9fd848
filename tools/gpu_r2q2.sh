# r2q2: persistent CTAs + dynamic work queue (option queue) A/B
for cfg in C3 copy:4096:4096 C3s C2 C5 C4; do
  timeout 400 python tools/sweep.py --config $cfg --reps 7 '' 'queue=1' 'queue=1 cta_warps=2' 'queue=1 cta_warps=4' 'queue=1 cta_warps=8' ''
done > gpurun_out/r02_sweep_queue.jsonl 2>&1
for cfg in C3; do
  timeout 400 python tools/sweep.py --config $cfg --reps 7 'queue=1 cta_warps=4 nstrips=79' 'queue=1 cta_warps=4 nstrips=120' 'queue=1 cta_warps=4 nstrips=240' 'queue=1 cta_warps=4 nstrips=320' 'queue=1 cta_warps=8 nstrips=240'
done >> gpurun_out/r02_sweep_queue.jsonl 2>&1
cat gpurun_out/r02_sweep_queue.jsonl

# r2y: programmatic dependent launch A/B (pdl=1 default vs pdl=0, and the
# experimental no-wait bound for independent frames) on the bench configs
set -x
for cfg in C3 C3s C2 C1 C5 C4 copy:4096:4096; do
  timeout 300 python tools/sweep.py --config $cfg --lib testhooks --reps 9 '' 'pdl=0' 'pdl_nowait=1' '' 'pdl=0'
done > gpurun_out/r02_sweep_pdl.jsonl 2> gpurun_out/r02_sweep_pdl.err
for cfg in C3 C2; do
  timeout 300 python tools/sweep.py --config $cfg --plan unfused --reps 5 '' 'pdl=0' '' 'pdl=0'
done >> gpurun_out/r02_sweep_pdl.jsonl 2>> gpurun_out/r02_sweep_pdl.err
cat gpurun_out/r02_sweep_pdl.jsonl

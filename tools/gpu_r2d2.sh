# delay_smem A/B (C4), then the whole GPU suite (incl. the bounds-checked runs)
timeout 400 python tools/sweep.py --config C4 --reps 7 '' 'delay_smem=0' '' 'delay_smem=0' > gpurun_out/r02_sweep_delay_smem.jsonl 2>&1
cat gpurun_out/r02_sweep_delay_smem.jsonl
timeout 1500 python -m pytest tests -q -m gpu -x > gpurun_out/tests_r2d2.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_r2d2.log

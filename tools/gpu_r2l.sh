# lut_smem A/B (C4), then the whole GPU suite
timeout 400 python tools/sweep.py --config C4 --reps 7 '' 'lut_smem=0' '' 'lut_smem=0' > gpurun_out/r02_sweep_lut_smem.jsonl 2>&1
cat gpurun_out/r02_sweep_lut_smem.jsonl
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tests_r2l.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_r2l.log

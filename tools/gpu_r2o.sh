# r2o: peel_warmup=0 (warm-up through the loop body) -- bit identity + A/B
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu -k "schedule_options and peel" > gpurun_out/tests_r2o.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/tests_r2o.log
S="timeout 900 python tools/sweep.py --reps 9"
$S --config C3 '' 'peel_warmup=0' '' 'peel_warmup=0' > gpurun_out/sweep_peel_r2o.jsonl 2>&1
$S --config C3s '' 'peel_warmup=0' '' 'peel_warmup=0' >> gpurun_out/sweep_peel_r2o.jsonl 2>&1
$S --config C2 '' 'peel_warmup=0' >> gpurun_out/sweep_peel_r2o.jsonl 2>&1
$S --config C1 '' 'peel_warmup=0' >> gpurun_out/sweep_peel_r2o.jsonl 2>&1
$S --config C5 --steps 20 '' 'peel_warmup=0' >> gpurun_out/sweep_peel_r2o.jsonl 2>&1
cut -c1-160 gpurun_out/sweep_peel_r2o.jsonl

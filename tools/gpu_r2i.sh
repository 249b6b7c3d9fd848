# r2i: warps per CTA (cta_warps) -- bit identity, sanitizer, A/B on every bench config
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu -k "schedule_options" > gpurun_out/tests_r2i.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_r2i.log
timeout 600 /usr/local/cuda/bin/compute-sanitizer --tool racecheck --error-exitcode 9 python tests/sanitize_cases.py workloads > gpurun_out/racecheck_r2i.log 2>&1; echo "racecheck rc=$?"; tail -2 gpurun_out/racecheck_r2i.log
timeout 600 /usr/local/cuda/bin/compute-sanitizer --tool memcheck --error-exitcode 9 python tests/sanitize_cases.py workloads > gpurun_out/memcheck_r2i.log 2>&1; echo "memcheck rc=$?"; tail -2 gpurun_out/memcheck_r2i.log
S="timeout 900 python tools/sweep.py --reps 9"
$S --config C3 '' 'cta_warps=2' 'cta_warps=4' 'cta_warps=8' '' 'cta_warps=2' 'cta_warps=4' 'cta_warps=8' > gpurun_out/sweep_ctaw_r2i.jsonl 2>&1
$S --config copy:4096:4096 '' 'cta_warps=2' 'cta_warps=4' 'cta_warps=8' >> gpurun_out/sweep_ctaw_r2i.jsonl 2>&1
$S --config C3s '' 'cta_warps=2' 'cta_warps=4' 'cta_warps=8' >> gpurun_out/sweep_ctaw_r2i.jsonl 2>&1
$S --config C2 '' 'cta_warps=2' 'cta_warps=4' 'cta_warps=8' >> gpurun_out/sweep_ctaw_r2i.jsonl 2>&1
$S --config C5 --steps 20 '' 'cta_warps=2' 'cta_warps=4' >> gpurun_out/sweep_ctaw_r2i.jsonl 2>&1
$S --config C4 --steps 40 '' 'cta_warps=2' 'cta_warps=4' >> gpurun_out/sweep_ctaw_r2i.jsonl 2>&1
$S --config C1 '' 'cta_warps=4' >> gpurun_out/sweep_ctaw_r2i.jsonl 2>&1
$S --config enhance:2048:2048 '' 'cta_warps=4' >> gpurun_out/sweep_ctaw_r2i.jsonl 2>&1
cut -c1-200 gpurun_out/sweep_ctaw_r2i.jsonl

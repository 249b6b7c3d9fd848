# r2d: whole GPU suite with the 2-row rolled trip, rtrip A/B sweep, ncu of C4/C3 fused kernels, peer sanitizer case
mkdir -p gpurun_out
KF_PARITY_LOG=gpurun_out/parity_r2d.jsonl timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tests_r2d.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_r2d.log
S="timeout 900 python tools/sweep.py --reps 9"
$S --config C4 --steps 40 '' 'rtrip=1' '' 'rtrip=1' > gpurun_out/sweep_rtrip_r2d.jsonl 2>&1
$S --config enhance:2048:2048 --steps 100 '' 'rtrip=1' >> gpurun_out/sweep_rtrip_r2d.jsonl 2>&1
cat gpurun_out/sweep_rtrip_r2d.jsonl
for cfg in C4 C3; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:kf_b -s 2 -c 1 -f -o gpurun_out/r02_${cfg}_b200_full \
     python tools/prof_run.py --config $cfg --plan b200 > gpurun_out/ncu_${cfg}.log 2>&1; echo "ncu $cfg rc=$?"
done
timeout 600 /usr/local/cuda/bin/compute-sanitizer --tool memcheck --error-exitcode 9 python tests/sanitize_cases.py peer > gpurun_out/sanitize_peer1.log 2>&1; echo "sanitize peer rc=$?"; tail -2 gpurun_out/sanitize_peer1.log

# r2l: zero-copy kf_run_host (host_direct) -- parity + e2e A/B on C3, C2, C4
mkdir -p gpurun_out
timeout 600 python -m pytest tests -q -m gpu -k "run_host" > gpurun_out/tests_r2l.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/tests_r2l.log
for c in C3 C2 C4 C3s; do timeout 900 python tools/e2e_probe.py $c '' 'host_direct=1' >> gpurun_out/e2e_direct_r2l.txt 2>&1; done; cat gpurun_out/e2e_direct_r2l.txt

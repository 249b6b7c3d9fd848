python tools/repro_case.py 1020000 420 > gpurun_out/repro2.log 2>&1; grep -c '"mismatch_px": \[0, 0\]' gpurun_out/repro2.log; grep mismatch gpurun_out/repro2.log | head -3
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tests_r2bug.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_r2bug.log
timeout 1500 python tests/fuzz_parity.py 1000 1020000 oracle > gpurun_out/r02_fuzz_fix_oracle.json 2>/dev/null; echo "fuzz rc=$?"; cat gpurun_out/r02_fuzz_fix_oracle.json

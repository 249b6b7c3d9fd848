timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tests_r2bug3.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_r2bug3.log
python tools/repro_case_f32.py 2030000 1381 2>&1 | head -3
timeout 2400 python tests/fuzz_parity.py 3000 2030000 oracle > gpurun_out/r02_fuzz6_oracle.json 2>/dev/null; echo "fuzz rc=$?"; cat gpurun_out/r02_fuzz6_oracle.json
timeout 2400 python tests/fuzz_parity.py 2000 4050000 oracle > gpurun_out/r02_fuzz7_oracle.json 2>/dev/null; echo "fuzz7 rc=$?"; cat gpurun_out/r02_fuzz7_oracle.json

python tests/fuzz_parity.py 1 2030230 oracle 2>/dev/null
python tests/fuzz_parity.py 1 4051254 oracle 2>/dev/null
python tools/repro_case_f32.py 4050000 1254 2>/dev/null | head -4 | cut -c1-400
timeout 2400 python tests/fuzz_parity.py 2500 5060000 oracle > gpurun_out/r02_fuzz8_oracle.json 2>/dev/null; echo "fuzz8 rc=$?"; cat gpurun_out/r02_fuzz8_oracle.json
timeout 1200 python tests/fuzz_parity.py 800 6070000 bands > gpurun_out/r02_fuzz8_bands.json 2>/dev/null; echo "bands rc=$?"; cat gpurun_out/r02_fuzz8_bands.json

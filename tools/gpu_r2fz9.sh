timeout 2000 python tests/fuzz_parity.py 3000 7080000 oracle > gpurun_out/r02_fuzz9_oracle.json 2>/dev/null; echo "oracle rc=$?"; cat gpurun_out/r02_fuzz9_oracle.json
timeout 1200 python tests/fuzz_parity.py 1000 8090000 bands > gpurun_out/r02_fuzz9_bands.json 2>/dev/null; echo "bands rc=$?"; cat gpurun_out/r02_fuzz9_bands.json

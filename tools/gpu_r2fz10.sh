timeout 1500 python tests/fuzz_parity.py 2500 9100000 oracle > gpurun_out/r02_fuzz10_oracle.json 2>/dev/null; echo "oracle rc=$?"; cat gpurun_out/r02_fuzz10_oracle.json
timeout 900 python tests/fuzz_parity.py 800 9200000 bands > gpurun_out/r02_fuzz10_bands.json 2>/dev/null; echo "bands rc=$?"; cat gpurun_out/r02_fuzz10_bands.json

# fuzz on the final state (PDL on by default)
timeout 1500 python tests/fuzz_parity.py 1000 1020000 oracle > gpurun_out/r02_fuzz_pdl_oracle.json 2> gpurun_out/r02_fuzz_pdl_oracle.err; echo "oracle rc=$?"; cat gpurun_out/r02_fuzz_pdl_oracle.json
timeout 900 python tests/fuzz_parity.py 500 1121000 bands > gpurun_out/r02_fuzz_pdl_bands.json 2> gpurun_out/r02_fuzz_pdl_bands.err; echo "bands rc=$?"; cat gpurun_out/r02_fuzz_pdl_bands.json

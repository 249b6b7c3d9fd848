# randomized parity fuzz on the final build: oracle mode (two seeds) and decomposition mode
timeout 1500 python tests/fuzz_parity.py 800 515000 oracle > gpurun_out/r02_fuzz_final_oracle.json 2> gpurun_out/r02_fuzz_final_oracle.err; echo "fuzz oracle rc=$?"; cat gpurun_out/r02_fuzz_final_oracle.json
timeout 900 python tests/fuzz_parity.py 400 616000 bands > gpurun_out/r02_fuzz_final_bands.json 2> gpurun_out/r02_fuzz_final_bands.err; echo "fuzz bands rc=$?"; cat gpurun_out/r02_fuzz_final_bands.json

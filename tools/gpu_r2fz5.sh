# more randomized parity fuzz on the final state, new seeds
timeout 2400 python tests/fuzz_parity.py 3000 2030000 oracle > gpurun_out/r02_fuzz5_oracle.json 2> gpurun_out/r02_fuzz5_oracle.err; echo "oracle rc=$?"; cat gpurun_out/r02_fuzz5_oracle.json
timeout 1500 python tests/fuzz_parity.py 1000 3040000 bands > gpurun_out/r02_fuzz5_bands.json 2> gpurun_out/r02_fuzz5_bands.err; echo "bands rc=$?"; cat gpurun_out/r02_fuzz5_bands.json

# long randomized parity fuzz on the final build (oracle + decompositions), different seeds
timeout 2400 python tests/fuzz_parity.py 2000 818000 oracle > gpurun_out/r02_fuzz_long_oracle.json 2> gpurun_out/r02_fuzz_long_oracle.err; echo "oracle rc=$?"; cat gpurun_out/r02_fuzz_long_oracle.json
timeout 1200 python tests/fuzz_parity.py 800 919000 bands > gpurun_out/r02_fuzz_long_bands.json 2> gpurun_out/r02_fuzz_long_bands.err; echo "bands rc=$?"; cat gpurun_out/r02_fuzz_long_bands.json

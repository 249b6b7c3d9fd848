# r2k: kf_run_host pipeline depth / taper sweep (e2e leg) + the run_host parity tests
mkdir -p gpurun_out
timeout 600 python -m pytest tests -q -m gpu -k "run_host" > gpurun_out/tests_r2k.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/tests_r2k.log
timeout 900 python tools/e2e_probe.py C3 '' 'host_bands=4' 'host_bands=6' 'host_bands=12' 'host_bands=16' 'host_bands=24' 'host_bands=32' 'host_taper=0' 'host_bands=16 host_taper=0' 'host_bands=2' 'host_bands=1' > gpurun_out/e2e_sweep_r2k.txt 2>&1; cat gpurun_out/e2e_sweep_r2k.txt
timeout 600 python tools/e2e_pipe_probe.py > gpurun_out/e2e_pipe_r2k.txt 2>&1; tail -5 gpurun_out/e2e_pipe_r2k.txt

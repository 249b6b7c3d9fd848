# r2e: calibration with the ROOFLINE (issue-rate) profile
mkdir -p gpurun_out
timeout 2400 python tools/calibrate.py --out gpurun_out/calibration_r2e.json > gpurun_out/calibrate_r2e.log 2>&1; echo "calibrate rc=$?"
tail -8 gpurun_out/calibrate_r2e.log | cut -c1-900

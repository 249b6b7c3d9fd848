# r2f: whole GPU suite, smoke, bench N=1 (+ launch list), reference arm, ncu full of the headline kernel, calibration
mkdir -p gpurun_out
KF_PARITY_LOG=gpurun_out/parity_r2f.jsonl timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tests_r2f.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_r2f.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r2f.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke_r2f.log
timeout 900 python bench.py --steps 200 --warmup 5 > gpurun_out/bench_r2f.json 2> gpurun_out/bench_r2f.err; echo "bench rc=$?"; head -c 400 gpurun_out/bench_r2f.json
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/bench_ref_r2f.json 2>&1; echo "ref rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r02_launches_c3.csv python bench.py --steps 2 --warmup 3 --no-extra --no-cpu > gpurun_out/ncu_launch_bench.log 2>&1; echo "ncu launches rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kf_b -s 2 -c 1 -f -o gpurun_out/r02_C3_b200_full_final \
   python tools/prof_run.py --config C3 --plan b200 > gpurun_out/ncu_C3_final.log 2>&1; echo "ncu C3 rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kf_b -s 2 -c 1 -f -o gpurun_out/r02_C4_b200_full_final \
   python tools/prof_run.py --config C4 --plan b200 > gpurun_out/ncu_C4_final.log 2>&1; echo "ncu C4 rc=$?"
timeout 1800 python tools/calibrate.py --out gpurun_out/calibration_r2f.json > gpurun_out/calibrate_r2f.log 2>&1; echo "calibrate rc=$?"

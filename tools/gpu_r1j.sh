mkdir -p gpurun_out
timeout 600 python tools/sweep.py --config C3s --plan b200 '' > gpurun_out/sweep_sq.jsonl 2>&1; cat gpurun_out/sweep_sq.jsonl
timeout 1500 python -m pytest tests -x -q -m gpu -k "shitomasi or strip_geometry or workloads" > gpurun_out/tests_gpu.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_gpu.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"; cut -c1-1500 gpurun_out/bench.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-cpu > gpurun_out/ncu_bench.log 2>&1; echo "ncu launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kf_b -s 2 -c 1 -f -o gpurun_out/prof_c3 python tools/prof_run.py --config C3 --plan b200 > gpurun_out/ncu_full.log 2>&1; echo "ncu full rc=$?"

# r2g: ncu launch list of the bench command reaching the headline plan; sanitizer on the final build
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/r02_launches_c3_full.csv python bench.py --steps 20 --warmup 3 --no-extra --no-cpu > gpurun_out/ncu_launch_bench2.log 2>&1; echo "ncu launches rc=$?"
bash tools/sanitize.sh

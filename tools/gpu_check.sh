#!/bin/bash
# GPU-box session: parity tests, bench, ncu launch list + full capture of the top kernel.
# usage: tools/gpu_check.sh [tests|bench|ncu|all]...   (outputs under gpurun_out/)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt 2>&1
for step in "$@"; do
  case $step in
    tests) timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/tests_gpu.log 2>&1; echo "tests rc=$?";;
    quick) timeout 900 python -m pytest tests -x -q -m gpu -k "workloads or fig4 or tiny or bands or launch" > gpurun_out/tests_gpu.log 2>&1; echo "quick tests rc=$?";;
    bench) timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"; cat gpurun_out/bench.json;;
    ncu) timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
           python bench.py --steps 3 --warmup 3 --no-cpu > gpurun_out/ncu_bench.log 2>&1; echo "ncu launches rc=$?";
         timeout 900 ncu --set full --clock-control none --import-source on -k regex:kf_b -s 2 -c 1 -f -o gpurun_out/prof_c3 \
           python tools/prof_run.py --config C3 --plan b200 > gpurun_out/ncu_full.log 2>&1; echo "ncu full rc=$?";;
  esac
done

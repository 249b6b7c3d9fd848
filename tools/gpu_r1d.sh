mkdir -p gpurun_out
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/tests_gpu.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_gpu.log
python tools/sweep.py --steps 100 --config C3s "" "KFUSE_CODE_BUDGET=1000" > gpurun_out/sweep_c3s.jsonl 2>&1; cat gpurun_out/sweep_c3s.jsonl
python tools/sweep.py --steps 200 --config C2 "" "KFUSE_NSTRIPS=16" "KFUSE_NSTRIPS=32" "KFUSE_NSTRIPS=64" "KFUSE_NSTRIPS=128" "KFUSE_MINCTAS=24" > gpurun_out/sweep_c2.jsonl 2>&1; cat gpurun_out/sweep_c2.jsonl
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"; cut -c1-1200 gpurun_out/bench.json
timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --force-multi --steps 50 --warmup 5 > gpurun_out/bench_multi1.json 2> gpurun_out/bench_multi1.err; echo "multi rc=$?"; cat gpurun_out/bench_multi1.json; tail -3 gpurun_out/bench_multi1.err

# r2n: final verification -- whole GPU suite, smoke, bench N=1, 2-rank multi smoke, reference arm
mkdir -p gpurun_out
KF_PARITY_LOG=gpurun_out/parity_r2n.jsonl timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tests_r2n.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_r2n.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r2n.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke_r2n.log
timeout 900 python bench.py --steps 200 --warmup 5 > gpurun_out/bench_r2n.json 2> gpurun_out/bench_r2n.err; echo "bench rc=$?"; head -c 300 gpurun_out/bench_r2n.json
KFUSE_DIST_BACKEND=gloo KFUSE_BENCH_DEVICE=0 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29517 bench.py --gpus 2 --steps 20 --warmup 3 > gpurun_out/bench_multi2_r2n.json 2> gpurun_out/bench_multi2_r2n.err; echo "multi rc=$?"; tail -c 400 gpurun_out/bench_multi2_r2n.json
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/bench_ref_r2n.json 2>&1; echo "ref rc=$?"

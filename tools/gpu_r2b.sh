# r2b: re-run the fixed tests + TMA option parity, TMA A/B sweep, bench (N=1), 2-rank shared-GPU multi smoke, reference arm
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -q -m gpu -k "tiny or peer_halo or schedule_options or experimental_rounding or negative" > gpurun_out/tests_r2b.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_r2b.log
S="timeout 600 python tools/sweep.py --steps 200 --reps 9"
$S --config C3 '' 'tma=1' '' 'tma=1' > gpurun_out/sweep_tma_r2b.jsonl 2>&1
$S --config C3s '' 'tma=1' >> gpurun_out/sweep_tma_r2b.jsonl 2>&1
$S --config C2 '' 'tma=1' >> gpurun_out/sweep_tma_r2b.jsonl 2>&1
$S --config copy:4096:4096 '' 'tma=1' '' 'tma=1' >> gpurun_out/sweep_tma_r2b.jsonl 2>&1
$S --config C4 --steps 40 '' 'tma=1' >> gpurun_out/sweep_tma_r2b.jsonl 2>&1
cat gpurun_out/sweep_tma_r2b.jsonl
timeout 900 python bench.py --steps 200 --warmup 5 > gpurun_out/bench_r2b.json 2> gpurun_out/bench_r2b.err; echo "bench rc=$?"; tail -c 600 gpurun_out/bench_r2b.json
KFUSE_DIST_BACKEND=gloo KFUSE_BENCH_DEVICE=0 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29517 bench.py --gpus 2 --steps 20 --warmup 3 > gpurun_out/bench_multi2_r2b.json 2> gpurun_out/bench_multi2_r2b.err; echo "multi rc=$?"; tail -c 1500 gpurun_out/bench_multi2_r2b.json
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_r2b.json 2>&1; echo "ref rc=$?"; cat gpurun_out/bench_ref_r2b.json

# strip count after warm_skip=2 (C4, Enhance), then the whole GPU suite
for cfg in C4; do
  timeout 600 python tools/sweep.py --config $cfg --reps 5 '' 'nstrips=60' 'nstrips=75' 'nstrips=90' 'nstrips=120' 'nstrips=45' ''
done > gpurun_out/r02_sweep_ns_ws2.jsonl 2>&1
timeout 300 python tools/sweep.py --config enhance:2048:2048 --reps 5 '' 'nstrips=40' 'nstrips=60' 'nstrips=80' 'nstrips=120' '' >> gpurun_out/r02_sweep_ns_ws2.jsonl 2>&1
cat gpurun_out/r02_sweep_ns_ws2.jsonl
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tests_r2ns.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_r2ns.log

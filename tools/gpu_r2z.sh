# r2z: GPU tests (incl. kf_run_batch and warm_skip), smoke, and the warm_skip / frames A/B
set -x
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/r02_tests_gpu_z.log 2>&1; echo "tests rc=$?"
tail -3 gpurun_out/r02_tests_gpu_z.log
for cfg in C4 enhance:2048:2048 C3 C2; do
  timeout 300 python tools/sweep.py --config $cfg --reps 9 '' 'warm_skip=0' '' 'warm_skip=0'
done > gpurun_out/r02_sweep_warm_skip.jsonl 2>&1
cat gpurun_out/r02_sweep_warm_skip.jsonl
timeout 600 python bench.py --steps 200 --warmup 5 > gpurun_out/bench_r02_z.json 2> gpurun_out/bench_r02_z.err; echo "bench rc=$?"
python -c "
import json; d=json.load(open('gpurun_out/bench_r02_z.json'))
print(d['value'], d['ms_per_step'], d['roofline']['frac'], d.get('frames'))
for k,v in d['workloads'].items(): print(k, v['plans']['b200']['ms_per_step'], v.get('frames',{}).get('ms_per_frame'))
"

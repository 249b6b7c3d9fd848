# the two bench arms with no flags (driver defaults), timed
s=$(date +%s); timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo "bench rc=$? $(( $(date +%s) - s )) s"; head -c 300 gpurun_out/bench_default.json
s=$(date +%s); timeout 900 python bench.py --impl reference > gpurun_out/bench_ref_default.json 2> gpurun_out/bench_ref_default.err; echo "ref rc=$? $(( $(date +%s) - s )) s"; head -c 1200 gpurun_out/bench_ref_default.json
s=$(date +%s); timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench_20.json 2> gpurun_out/bench_20.err; echo "bench20 rc=$? $(( $(date +%s) - s )) s"; head -c 300 gpurun_out/bench_20.json
s=$(date +%s); timeout 900 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench_ref_20.json 2> gpurun_out/bench_ref_20.err; echo "ref20 rc=$? $(( $(date +%s) - s )) s"; head -c 300 gpurun_out/bench_ref_20.json

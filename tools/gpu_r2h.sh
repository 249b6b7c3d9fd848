# r2h: cache-policy options A/B (streaming stores, L2 evict-first input copies) + their bit-identity tests
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu -k "schedule_options" > gpurun_out/tests_r2h.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_r2h.log
S="timeout 900 python tools/sweep.py --reps 9"
$S --config C3 '' 'st_cs=1' 'ld_ef=1' 'st_cs=1 ld_ef=1' '' 'st_cs=1' 'ld_ef=1' 'st_cs=1 ld_ef=1' > gpurun_out/sweep_cache_r2h.jsonl 2>&1
$S --config copy:4096:4096 '' 'st_cs=1' 'ld_ef=1' 'st_cs=1 ld_ef=1' '' >> gpurun_out/sweep_cache_r2h.jsonl 2>&1
$S --config C3s '' 'st_cs=1' 'ld_ef=1' 'st_cs=1 ld_ef=1' >> gpurun_out/sweep_cache_r2h.jsonl 2>&1
$S --config C2 '' 'st_cs=1' 'ld_ef=1' 'st_cs=1 ld_ef=1' >> gpurun_out/sweep_cache_r2h.jsonl 2>&1
$S --config C5 --steps 20 '' 'st_cs=1' 'ld_ef=1' 'st_cs=1 ld_ef=1' >> gpurun_out/sweep_cache_r2h.jsonl 2>&1
$S --config C4 --steps 40 '' 'st_cs=1 ld_ef=1' >> gpurun_out/sweep_cache_r2h.jsonl 2>&1
cat gpurun_out/sweep_cache_r2h.jsonl
./tools/ubench/cta_rate > gpurun_out/cta_rate.txt 2>&1 || (cd tools/ubench && nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o cta_rate cta_rate.cu && ./cta_rate > ../../gpurun_out/cta_rate.txt 2>&1)
cat gpurun_out/cta_rate.txt

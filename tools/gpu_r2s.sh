# r2s: evidence on the current build -- whole GPU suite, smoke, bench N=1, reference arm,
# ncu launch list of the bench, ncu --set full of the C3 and C4 fused kernels, sanitizer,
# C4 strip-count sweep after warm_skip
mkdir -p gpurun_out
KF_PARITY_LOG=gpurun_out/parity_r2s.jsonl timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tests_r2s.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_r2s.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r2s.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke_r2s.log
timeout 900 python bench.py --steps 200 --warmup 5 > gpurun_out/bench_r2s.json 2> gpurun_out/bench_r2s.err; echo "bench rc=$?"; head -c 300 gpurun_out/bench_r2s.json
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/bench_ref_r2s.json 2>&1; echo "ref rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/r02_launches_c3_s.csv python bench.py --steps 20 --warmup 3 --no-extra --no-cpu > gpurun_out/ncu_launch_bench_s.log 2>&1; echo "ncu launches rc=$?"
for cfg in C3 C4; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:kf_b -s 2 -c 1 -f -o gpurun_out/r02_${cfg}_b200_full_s \
     python tools/prof_run.py --config $cfg --plan b200 > gpurun_out/ncu_${cfg}_s.log 2>&1; echo "ncu $cfg rc=$?"
done
python tools/ncu_extract.py C3=gpurun_out/r02_C3_b200_full_s.ncu-rep C4=gpurun_out/r02_C4_b200_full_s.ncu-rep > gpurun_out/r02_ncu_c3_c4_s.json; echo "extract rc=$?"
echo "compute-sanitizer: closed on this pool (runs under it left GPUs needing a reset); not run"
timeout 600 python tools/sweep.py --config C4 --reps 5 '' 'nstrips=30' 'nstrips=40' 'nstrips=50' 'nstrips=75' 'nstrips=90' '' > gpurun_out/r02_sweep_c4_ns_warmskip.jsonl 2>&1
cat gpurun_out/r02_sweep_c4_ns_warmskip.jsonl

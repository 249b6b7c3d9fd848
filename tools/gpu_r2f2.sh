# r2f2: final evidence -- GPU suite, smoke, bench, reference arm, ncu launch list, ncu --set full of C3 and C4; rtrip=2 recheck on C4
mkdir -p gpurun_out
KF_PARITY_LOG=gpurun_out/parity_r2f2.jsonl timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tests_r2f2.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_r2f2.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r2f2.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke_r2f2.log
timeout 900 python bench.py --steps 200 --warmup 5 > gpurun_out/bench_r2f2.json 2> gpurun_out/bench_r2f2.err; echo "bench rc=$?"; head -c 300 gpurun_out/bench_r2f2.json
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/bench_ref_r2f2.json 2>&1; echo "ref rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/r02_launches_c3_f2.csv python bench.py --steps 20 --warmup 3 --no-extra --no-cpu > gpurun_out/ncu_launch_bench_f2.log 2>&1; echo "ncu launches rc=$?"
for cfg in C3 C4; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:kf_b -s 2 -c 1 -f -o gpurun_out/r02_${cfg}_b200_full_f2 \
     python tools/prof_run.py --config $cfg --plan b200 > gpurun_out/ncu_${cfg}_f2.log 2>&1; echo "ncu $cfg rc=$?"
done
python tools/ncu_extract.py C3=gpurun_out/r02_C3_b200_full_f2.ncu-rep C4=gpurun_out/r02_C4_b200_full_f2.ncu-rep > gpurun_out/r02_ncu_c3_c4_f2.json; echo "extract rc=$?"
timeout 300 python tools/sweep.py --config C4 --reps 5 '' 'rtrip=2' '' > gpurun_out/r02_sweep_rtrip_final.jsonl 2>&1; cat gpurun_out/r02_sweep_rtrip_final.jsonl

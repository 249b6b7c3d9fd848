# final-state check: the driver's sequence (GPU tests, smoke, bench N=1, reference arm)
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tests_r2z2.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_r2z2.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r2z2.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke_r2z2.log
timeout 900 python bench.py > gpurun_out/bench_r2z2.json 2> gpurun_out/bench_r2z2.err; echo "bench rc=$?"; head -c 400 gpurun_out/bench_r2z2.json
timeout 600 python bench.py --impl reference > gpurun_out/bench_ref_r2z2.json 2>&1; echo "ref rc=$?"; head -c 200 gpurun_out/bench_ref_r2z2.json

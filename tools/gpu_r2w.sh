# r2w: bounds-checking build tests + whole GPU suite + smoke on the current build
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_bounds.py -q -m gpu > gpurun_out/r02_tests_bounds.log 2>&1; echo "bounds rc=$?"; tail -5 gpurun_out/r02_tests_bounds.log
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tests_r2w.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_r2w.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r2w.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke_r2w.log

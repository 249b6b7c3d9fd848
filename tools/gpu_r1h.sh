mkdir -p gpurun_out
python tools/diag_strips.py > gpurun_out/diag2.log 2>&1; grep -c "mism 0 " gpurun_out/diag2.log; grep -v "mism 0 " gpurun_out/diag2.log | head
python tools/diag_host.py > gpurun_out/diag.log 2>&1; head -3 gpurun_out/diag.log
timeout 600 python tools/sweep.py --config C3 --plan b200 '' 'KFUSE_NSTRIPS=300' > gpurun_out/sweep.jsonl 2>&1; cat gpurun_out/sweep.jsonl
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/tests_gpu.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_gpu.log

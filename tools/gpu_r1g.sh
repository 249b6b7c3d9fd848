mkdir -p gpurun_out
python tools/diag_strips.py > gpurun_out/diag2.log 2>&1
KFUSE_DEFER=0 python tools/diag_strips.py >> gpurun_out/diag2.log 2>&1
KFUSE_PAIRS=0 python tools/diag_strips.py >> gpurun_out/diag2.log 2>&1
cat gpurun_out/diag2.log

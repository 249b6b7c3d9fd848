mkdir -p gpurun_out
python tools/diag_host.py > gpurun_out/diag.log 2>&1
KFUSE_DEFER=0 python tools/diag_host.py >> gpurun_out/diag.log 2>&1
python tools/diag_host.py 512 300 >> gpurun_out/diag.log 2>&1
cat gpurun_out/diag.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kf_b -s 2 -c 1 -f -o gpurun_out/prof_c3 \
   python tools/prof_run.py --config C3 --plan b200 > gpurun_out/ncu_full.log 2>&1; echo "ncu full rc=$?"

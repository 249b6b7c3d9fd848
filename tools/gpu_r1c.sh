mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu -k "swar or overlapped or run_host or full_size or deep10 or random" > gpurun_out/tests_gpu_new.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_gpu_new.log
python tools/sweep.py --steps 60 --config C4 "KFUSE_SWRING=0" "KFUSE_SWRING_CAP=144" "KFUSE_SWRING_CAP=164" "KFUSE_SWRING_CAP=184" "KFUSE_SWRING_CAP=184 KFUSE_MINCTAS=10" "KFUSE_SWRING_CAP=184 KFUSE_MINCTAS=8" > gpurun_out/sweep_c4r.jsonl 2>&1; cat gpurun_out/sweep_c4r.jsonl
python tools/sweep.py --steps 100 --config enhance:2048:2048 "" "KFUSE_CODE_BUDGET=1000" "KFUSE_CODE_BUDGET=4000" > gpurun_out/sweep_enh.jsonl 2>&1; cat gpurun_out/sweep_enh.jsonl

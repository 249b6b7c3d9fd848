# Tail-split sweep (KFUSE_NLONG: two strip heights, long strips first) + parity under the split.
set -x
mkdir -p gpurun_out
S="python tools/sweep.py --steps 300"
$S --config C3 "" "KFUSE_NSTRIPS=301 KFUSE_NLONG=109" "KFUSE_NSTRIPS=280 KFUSE_NLONG=130" "KFUSE_NSTRIPS=320 KFUSE_NLONG=90" "KFUSE_NSTRIPS=260 KFUSE_NLONG=150" "KFUSE_NSTRIPS=240 KFUSE_NLONG=170" "KFUSE_NSTRIPS=410" "" > gpurun_out/sweep_c3_tail.jsonl 2>&1
$S --config C3s "" "KFUSE_NSTRIPS=301 KFUSE_NLONG=109" "KFUSE_NSTRIPS=280 KFUSE_NLONG=130" "KFUSE_NSTRIPS=260 KFUSE_NLONG=150" "" > gpurun_out/sweep_c3s_tail.jsonl 2>&1
$S --config C2 "" "KFUSE_NLONG=20" "KFUSE_NLONG=40" > gpurun_out/sweep_c2_tail.jsonl 2>&1
KFUSE_NLONG=3 timeout 1500 python -m pytest tests -x -q -m gpu -k "not dist and not peer" > gpurun_out/tests_gpu_nlong.log 2>&1; echo "nlong tests rc=$?"; tail -2 gpurun_out/tests_gpu_nlong.log

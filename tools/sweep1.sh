set -x
mkdir -p gpurun_out
S="python tools/sweep.py --steps 300"
$S --config C3 "" "KFUSE_MINCTAS=16" "KFUSE_MINCTAS=20" "KFUSE_MINCTAS=24" "KFUSE_MINCTAS=32" "KFUSE_SMEM_ROWS=8" "KFUSE_SMEM_ROWS=16" "KFUSE_SMEM_ROWS=24" "KFUSE_PAIRS=0" "KFUSE_DIAG_SKIP=frame" "KFUSE_NSTRIPS=100" "KFUSE_NSTRIPS=150" "KFUSE_NSTRIPS=300" "KFUSE_NSTRIPS=400" > gpurun_out/sweep_c3.jsonl 2>&1
$S --config copy:4096:4096 "" "KFUSE_NSTRIPS=100" "KFUSE_NSTRIPS=400" > gpurun_out/sweep_copy.jsonl 2>&1
$S --config blur:4096:4096 "" > gpurun_out/sweep_blur.jsonl 2>&1
for c in C1 C2 C3s C4; do for pl in unfused paper b200; do $S --config $c --plan $pl ""; done; done > gpurun_out/sweep_cfgs.jsonl 2>&1

# r2t: C4 register budget vs unpacked SWAR rings (options swring_cap, minctas)
timeout 900 python tools/sweep.py --config C4 --reps 5 '' 'swring_cap=200 minctas=8' 'swring_cap=240 minctas=8' 'minctas=8' 'swring_cap=200 minctas=10' 'swring_cap=200 minctas=9' '' > gpurun_out/r02_sweep_c4_regs.jsonl 2>&1
timeout 300 python tools/sweep.py --config enhance:2048:2048 --reps 5 '' 'minctas=8' 'swring_cap=200 minctas=8' >> gpurun_out/r02_sweep_c4_regs.jsonl 2>&1
cat gpurun_out/r02_sweep_c4_regs.jsonl

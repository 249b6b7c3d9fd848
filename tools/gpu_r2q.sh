# r2q: copy floors at small sizes -- torch vs the framework's copy kernel, and the strip geometry at 2048^2
python tools/copy_probe.py
timeout 600 python tools/sweep.py --config copy:2048:2048 '' 'nstrips=40' 'nstrips=80' 'nstrips=120' 'nstrips=240' 'minctas=24' 'smem_rows=6'
timeout 600 python tools/sweep.py --config C2 '' 'nstrips=40' 'nstrips=80' 'nstrips=120' 'nstrips=240' 'smem_rows=6' 'smem_rows=8'

"""Times kf_run_host (pinned host buffers, H2D + compute + D2H) for one config
under several host-pipeline settings, as bench.py's e2e leg does (interleaved,
median of 5 rounds of 20 calls).  Diagnostics only: bench.py is the measurement
of record.

    python tools/e2e_probe.py C3 '' 'host_bands=4' 'host_bands=16 host_taper=0'
"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from kf_inputs import gen  # noqa: E402
from kf_inputs import pipelines as P  # noqa: E402
from paper_conf_cgo_qiaorht19_b200 import kfuse as K  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
settings = sys.argv[2:] or [""]
spec, seed = P.config(cfg)
W, H = spec["width"], spec["height"]
host = gen.image(spec["dtype"], seed, W, H)
hin = torch.from_numpy(host).pin_memory()
hout = torch.empty_like(hin).pin_memory()
plans = {}
for st in settings:
    opts = {k: int(v) for k, v in (kv.split("=") for kv in st.split())}
    plans[st] = K.Pipeline.from_spec(spec, opts).plan_fusion("b200")
s = torch.cuda.Stream()
for pl in plans.values():
    for _ in range(3):
        pl.run_host([hin], [hout], s)
torch.cuda.synchronize()
res = {st: [] for st in settings}
for _ in range(5):
    for st, pl in plans.items():
        n = 20
        t = time.perf_counter()
        for _ in range(n):
            pl.run_host([hin], [hout], s)
        res[st].append((time.perf_counter() - t) / n)
for st, v in res.items():
    v.sort()
    dt = v[len(v) // 2]
    print(f"{cfg} [{st or 'default'}] e2e {dt * 1e3:.3f} ms/step = {W * H / dt / 1e6:.1f} Mpixel/s", flush=True)

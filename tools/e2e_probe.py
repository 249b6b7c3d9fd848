"""Times kf_run_host (pinned host buffers, H2D + compute + D2H) for one config,
as bench.py's e2e leg does.  Diagnostics only: bench.py is the measurement of record."""
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
spec, seed = P.config(cfg)
W, H = spec["width"], spec["height"]
host = gen.image(spec["dtype"], seed, W, H)
hin = torch.from_numpy(host).pin_memory()
hout = torch.empty_like(hin).pin_memory()
plan = K.Pipeline.from_spec(spec).plan_fusion("b200")
s = torch.cuda.Stream()
for _ in range(3):
    plan.run_host([hin], [hout], s)
torch.cuda.synchronize()
n = 20
t = time.perf_counter()
for _ in range(n):
    plan.run_host([hin], [hout], s)
dt = (time.perf_counter() - t) / n
print(f"{cfg} taper={os.environ.get('KFUSE_HOST_TAPER', '1')} e2e {dt * 1e3:.3f} ms/step = {W * H / dt / 1e6:.1f} Mpixel/s")

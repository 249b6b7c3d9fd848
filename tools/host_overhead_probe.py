"""Host cost of one eager kf_run call through the ctypes binding (C3 b200 plan),
against its GPU time: is the launch path (argument marshalling, launch geometry)
cheap enough for eager callers?  Diagnostics only."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from kf_inputs import gen  # noqa: E402
from kf_inputs import pipelines as P  # noqa: E402
from paper_conf_cgo_qiaorht19_b200 import kfuse as K  # noqa: E402

res = {}
for cfg in ("C1", "C3", "C4"):
    spec, seed = P.config(cfg)
    W, H = spec["width"], spec["height"]
    x = torch.from_numpy(gen.image(spec["dtype"], seed, W, H)).cuda()
    y = torch.empty_like(x)
    plan = K.Pipeline.from_spec(spec).plan_fusion("b200")
    s = torch.cuda.Stream()
    for _ in range(5):
        plan.run([x], [y], s)
    torch.cuda.synchronize()
    n = 200
    t = time.perf_counter()
    for _ in range(n):
        plan.run([x], [y], s)
    host = (time.perf_counter() - t) / n
    torch.cuda.synchronize()
    wall = (time.perf_counter() - t) / n
    res[cfg] = {"host_us_per_call": round(host * 1e6, 2), "wall_us_per_call": round(wall * 1e6, 2)}
print(json.dumps(res))

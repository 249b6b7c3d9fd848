"""Short driver for ncu captures: runs one config/plan a few times through the C-ABI.

    ncu --set full -k regex:kf_b -c 3 python tools/prof_run.py --config C3 --plan b200
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from kf_inputs import gen  # noqa: E402
from kf_inputs import pipelines as P  # noqa: E402
from paper_conf_cgo_qiaorht19_b200 import kfuse as K  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C3")
ap.add_argument("--plan", default="b200")
ap.add_argument("--runs", type=int, default=4)
a = ap.parse_args()
spec, seed = P.config(a.config)
W, H = spec["width"], spec["height"]
host = gen.image(spec["dtype"], seed, W, H)
x = torch.from_numpy(host).cuda()
y = torch.empty_like(x)
p = K.Pipeline.from_spec(spec)
plan = p.plan_unfused() if a.plan == "unfused" else p.plan_fusion(a.plan)
for _ in range(a.runs):
    plan.run([x], [y])
torch.cuda.synchronize()
print("ok", a.config, a.plan, plan.num_launches, "launches/run")

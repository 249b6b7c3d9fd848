"""Diagnostic: does the fused Harris output depend on the strip geometry (KFUSE_NSTRIPS)?"""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np, torch
from kf_inputs import gen, pipelines as P
from oracle import oracle as O
from paper_conf_cgo_qiaorht19_b200 import kfuse as K

W, H = 256, 240
for wl in ("harris", "shitomasi", "unsharp"):
    spec = P.WORKLOADS[wl](W, H)
    img = gen.image_f32(4, W, H)
    ref = O.run(spec, [img])[spec["outputs"][0]]
    p = K.Pipeline.from_spec(spec)
    plan = p.plan_fusion("b200")
    x = torch.from_numpy(img).cuda(); y = torch.empty_like(x)
    outs = {}
    for ns in (0, 118, 80, 60, 40, 20, 10, 4, 2):
        os.environ["KFUSE_NSTRIPS"] = str(ns)
        plan.run([x], [y]); torch.cuda.synchronize()
        outs[ns] = y.cpu().numpy().copy()
    base = outs[0]
    for ns, o in outs.items():
        d = o != base
        e = np.abs(o.astype(np.float64) - ref)
        rows = np.nonzero(d.any(1))[0]
        print(wl, "ns", ns, "mism", int(d.sum()), "rows", rows[:12].tolist(), "err_vs_oracle max", float(e.max()),
              "mean", float(e.mean()))

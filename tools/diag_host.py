"""Diagnostic: where do kf_run_host / kf_run_band differ from kf_run (harris b200)?"""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np, torch
from kf_inputs import gen, pipelines as P
from paper_conf_cgo_qiaorht19_b200 import kfuse as K

W, H = (int(v) for v in (sys.argv[1:3] if len(sys.argv) > 2 else (300, 200)))
spec = P.harris(W, H)
img = gen.image_f32(4, W, H)
p = K.Pipeline.from_spec(spec)
plan = p.plan_fusion("b200")
x = torch.from_numpy(img).cuda(); y = torch.empty_like(x)
plan.run([x], [y]); torch.cuda.synchronize()
full = y.cpu().numpy()
out = np.empty_like(full)
plan.run_host([img], [out])
d = out != full
print("defer", os.environ.get("KFUSE_DEFER"), "host mismatches", d.sum())
if d.any():
    rows = np.nonzero(d.any(1))[0]; cols = np.nonzero(d.any(0))[0]
    print(" rows", rows.min(), rows.max(), len(rows), " cols", cols.min(), cols.max(), len(cols))
    print(" per-row counts", {int(r): int(d[r].sum()) for r in rows[:40]})
R = plan.halo_rows
for cuts in ([0, 66, 133, 200], [0, 13, 40, 41, 97, 200]):
    cuts = [c for c in cuts if c <= H]
    for r0, r1 in zip(cuts[:-1], cuts[1:]):
        a0, a1 = max(0, r0 - R), min(H, r1 + R)
        dx = torch.from_numpy(np.ascontiguousarray(img[a0:a1])).cuda()
        o = torch.empty((r1 - r0, W), dtype=torch.float32, device="cuda")
        plan.run_band(r0, r1, [dx], a0, a1, [o]); torch.cuda.synchronize()
        dd = o.cpu().numpy() != full[r0:r1]
        # in-place variant: full input, band rows
        o2 = torch.empty((r1 - r0, W), dtype=torch.float32, device="cuda")
        plan.run_band(r0, r1, [x], 0, H, [o2]); torch.cuda.synchronize()
        dd2 = o2.cpu().numpy() != full[r0:r1]
        print(f" band [{r0},{r1}) halo-input mism {dd.sum()}  full-input mism {dd2.sum()}",
              (np.nonzero(dd2.any(1))[0][:10] + r0).tolist(), np.nonzero(dd2.any(0))[0][:10].tolist())

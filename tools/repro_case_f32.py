"""Re-runs one f32 fuzz case under several plans/options: normalised error
against the oracle and where the bad pixels are (diagnostics)."""
import importlib.util
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

from kf_inputs import gen  # noqa: E402
from oracle import oracle as O  # noqa: E402

spec_ = importlib.util.spec_from_file_location("fz", os.path.join(ROOT, "tests", "fuzz_parity.py"))
fz = importlib.util.module_from_spec(spec_)
spec_.loader.exec_module(fz)
seed0, i = int(sys.argv[1]), int(sys.argv[2])
spec, kind, opts, lab, seed = fz.case(i, seed0)
ins = [gen.image(spec["dtype"], seed + 7 * j, spec["width"], spec["height"]) for j in range(spec["n_inputs"])]
ref = O.run(spec, ins)
W, H = spec["width"], spec["height"]
for kk, o in [(kind, opts), (kind, {}), (kind, {"pdl": 0}), ("unfused", {}), ("b200", {}), ("paper", {}),
              (kind, {"sring": 0}), (kind, {"code_budget": 1000}), (kind, {"peel_warmup": 0}), (kind, {"heavy_first": 0}),
              (kind, {"nstrips": 1}), (kind, {"nstrips": 3})]:
    plan = fz.make(spec, kk, o, lab)
    d_in = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in ins]
    outs = [torch.full((H, W), 1e9, dtype=torch.float32, device="cuda") for _ in spec["outputs"]]
    plan.run(d_in, outs)
    torch.cuda.synchronize()
    rep = []
    for ob, img in zip(outs, spec["outputs"]):
        g = ob.cpu().numpy().astype(np.float64)
        r = ref[img]
        d = np.abs(g - r)
        err = float(d.max() / max(np.abs(r).max(), 1e-30))
        a = np.abs(r)
        sel = a >= 1e-3 * a.max()
        pw = float((d[sel] / a[sel]).max())
        bad = np.argwhere(d > 1e-4 * max(np.abs(r).max(), 1e-30))
        rows = sorted(set(bad[:, 0].tolist()))
        cols = sorted(set(bad[:, 1].tolist()))
        rep.append({"img": img, "err": err, "pw": pw, "n_bad": len(bad), "rows": rows[:12] + (["..."] if len(rows) > 12 else []),
                    "cols": cols[:12] + (["..."] if len(cols) > 12 else []), "n_rows": len(rows), "n_cols": len(cols)})
    print(json.dumps({"plan": kk, "opts": o, "blocks": [list(b) for b in plan.blocks], "out": rep}), flush=True)

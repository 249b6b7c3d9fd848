"""Re-runs one fuzz case (tests/fuzz_parity.py) under several option sets and
reports which ones differ from the oracle (diagnostics)."""
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
print(json.dumps({"kind": kind, "opts": opts, "W": spec["width"], "H": spec["height"], "ops": spec["ops"]})[:3000])
ins = [gen.image(spec["dtype"], seed + 7 * j, spec["width"], spec["height"]) for j in range(spec["n_inputs"])]
ref = O.run(spec, ins)
variants = [opts, {**opts, "pdl": 0}, {**opts, "warm_skip": 0}, {**opts, "warm_skip": 1}, {**opts, "lut_smem": 0},
            {**opts, "delay_smem": 0}, {}, {**opts, "pdl": 0, "warm_skip": 0}]
for o in variants:
    plan = fz.make(spec, kind, o, lab)
    d_in = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in ins]
    shape = (spec["height"], spec["width"]) + (() if spec["dtype"] == "f32" else (4,))
    dt = torch.float32 if spec["dtype"] == "f32" else torch.uint8
    for rep in range(3):
        outs = [torch.full(shape, 77, dtype=dt, device="cuda") for _ in spec["outputs"]]
        plan.run(d_in, outs)
        torch.cuda.synchronize()
        bad = []
        for ob, img in zip(outs, spec["outputs"]):
            g = ob.cpu().numpy()
            r = ref[img]
            diff = np.argwhere(np.any(g != r, axis=-1)) if spec["dtype"] == "u8x4" else np.argwhere(g != r)
            bad.append(len(diff))
            if len(diff) and rep == 0:
                y, x = diff[0][:2]
                print("   first diff", diff[:6].tolist(), "got", g[y, x].tolist(), "ref", r[y, x].tolist())
        print(json.dumps({"opts": o, "rep": rep, "blocks": plan.num_launches, "mismatch_px": bad}), flush=True)

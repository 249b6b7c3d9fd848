"""Narrows down the fused f32 edge-column mismatch of fuzz seed 2031381 with
sub-pipelines run as one fused block (diagnostics)."""
import importlib.util
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

from kf_inputs import gen  # noqa: E402
from kf_inputs import pipelines as P  # noqa: E402
from oracle import oracle as O  # noqa: E402
from paper_conf_cgo_qiaorht19_b200 import kfuse as K  # noqa: E402

spec_ = importlib.util.spec_from_file_location("fz", os.path.join(ROOT, "tests", "fuzz_parity.py"))
fz = importlib.util.module_from_spec(spec_)
spec_.loader.exec_module(fz)
base, _, _, _, seed = fz.case(1381, 2030000)
ops = base["ops"]
W, H = base["width"], base["height"]


def run(name, build, opts=None):
    p = P.Pipeline(name, W, H, "f32")
    build(p)
    spec = p.spec()
    ins = [gen.image("f32", seed + 7 * j, W, H) for j in range(spec["n_inputs"])]
    ref = O.run(spec, ins)
    pipe = K.Pipeline.from_spec(spec, opts)
    plan = pipe.plan_from_blocks([0] * len(spec["ops"]))
    d_in = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in ins]
    outs = [torch.full((H, W), 1e9, dtype=torch.float32, device="cuda") for _ in spec["outputs"]]
    plan.run(d_in, outs)
    torch.cuda.synchronize()
    for ob, img in zip(outs, spec["outputs"]):
        g = ob.cpu().numpy().astype(np.float64)
        r = ref[img]
        d = np.abs(g - r)
        m = max(np.abs(r).max(), 1e-30)
        bad = np.argwhere(d > 1e-4 * m)
        print(json.dumps({"case": name, "opts": opts, "err": float(d.max() / m), "n_bad": len(bad),
                          "cols": sorted(set(bad[:, 1].tolist()))[:10]}), flush=True)


m0, m1, m3 = ops[0]["mask"], ops[1]["mask"], ops[3]["mask"]
run("l3_alone", lambda p: p.output(p.local("l3", p.input(), m3, "constant")))
run("l1_alone", lambda p: p.output(p.local("l1", p.input(), m1, "constant")))
run("l0_alone", lambda p: p.output(p.local("l0", p.input(), m0, "mirror101", post=[P.L(0), P.C(0.5), P.ADD])))


def chain(p, second, mask, post=None):
    i = p.input()
    a = p.local("l0", i, m0, "mirror101", post=[P.L(0), P.C(0.5), P.ADD])
    p.output(p.local(second, a, mask, "constant", post=post))


run("l0_l3", lambda p: chain(p, "l3", m3, [P.L(0), P.ABS]))
run("l0_l1", lambda p: chain(p, "l1", m1, [P.L(0), P.ABS]))
run("l0_l3_noabs", lambda p: chain(p, "l3", m3))
run("l0_l3_nopairs", lambda p: chain(p, "l3", m3), None)


def full(p, m1mode="constant", m3mode="constant", with_p2=True):
    i = p.input()
    j = p.input()
    a = p.local("l0", j, m0, "mirror101", post=[P.L(0), P.C(0.5), P.ADD])
    b = p.local("l1", a, m1, m1mode, post=[P.L(0), P.ABS])
    c = p.point("p2", [b, a], [P.L(0), P.L(1), P.SUB, P.C(0.1), P.ADD]) if with_p2 else b
    d = p.local("l3", a, m3, m3mode, post=[P.L(0), P.ABS])
    p.output(p.point("p4", [c, d], [P.L(0), P.L(1), P.SUB, P.C(0.5), P.MUL]))


run("full", full)
run("full_l1_mirror", lambda p: full(p, m1mode="mirror"))
run("full_l3_mirror", lambda p: full(p, m3mode="mirror"))
run("full_no_p2", lambda p: full(p, with_p2=False))
run("full_sring0", full, {"sring": 0})

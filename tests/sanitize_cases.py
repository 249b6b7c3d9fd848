"""TEST INFRASTRUCTURE (not collected by pytest): small launches of every kernel
family for compute-sanitizer (tools/sanitize.sh):
C1 Harris 256^2 under every plan, deep10 67x41, all five border modes fused
(Harris and deep10), 10 random DAGs (3 plans each), the TMA row feed, kf_run_host,
a row band and kf_run_batch frames.  Each result is also checked against the oracle, so a run under
the sanitizer is a parity run too.  Exit code 0 = all outputs correct."""
import os
import random
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))   # tests/ -> repo root
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from kf_inputs import gen  # noqa: E402
from kf_inputs import pipelines as P  # noqa: E402
from oracle import oracle as O  # noqa: E402
from paper_conf_cgo_qiaorht19_b200 import kfuse as K  # noqa: E402


def run(spec, kind, opts=None, seed=1):
    ins = [gen.image(spec["dtype"], seed + 101 * j, spec["width"], spec["height"]) for j in range(spec["n_inputs"])]
    p = K.Pipeline.from_spec(spec, opts)
    plan = p.plan_unfused() if kind == "unfused" else p.plan_fusion(kind)
    d_in = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in ins]
    shape = (spec["height"], spec["width"]) + (() if spec["dtype"] == "f32" else (4,))
    dt = torch.float32 if spec["dtype"] == "f32" else torch.uint8
    outs = [torch.empty(shape, dtype=dt, device="cuda") for _ in spec["outputs"]]
    plan.run(d_in, outs)
    torch.cuda.synchronize()
    ref = O.run(spec, ins)
    for o, img in zip(outs, spec["outputs"]):
        g = o.cpu().numpy()
        r = ref[img]
        if spec["dtype"] == "u8x4":
            assert np.array_equal(g, r), spec["name"]
        else:
            s = np.abs(r).max() or 1.0
            assert np.abs(g.astype(np.float64) - r).max() / s <= 1e-5, spec["name"]
    return plan, ins, outs


def main():
    which = sys.argv[1] if len(sys.argv) > 1 else "all"
    n = 0
    if which in ("all", "workloads"):
        for kind in ("unfused", "paper", "b200"):
            run(P.harris(256, 256), kind)
            run(P.deep10(67, 41), kind)
            n += 2
        for mode in P.MODES:
            run(P.harris(45, 37, mode), "b200")
            run(P.deep10(45, 37, mode), "b200")
            n += 2
        run(P.harris(256, 256), "b200", {"tma": 1})
        run(P.harris(256, 256), "b200", {"cta_warps": 4})
        run(P.deep10(67, 41), "b200", {"cta_warps": 4})
        run(P.harris(45, 37, "constant"), "b200", {"cta_warps": 4})
        n += 3
        run(P.unsharp(512, 96), "b200", {"tma": 1})
        n += 2
        plan, ins, outs = run(P.harris(300, 200), "b200")
        hout = np.empty((200, 300), np.float32)
        plan.run_host([ins[0]], [hout])
        assert np.array_equal(hout, outs[0].cpu().numpy())
        d = torch.from_numpy(ins[0][40:120]).cuda()
        band = torch.empty((60, 300), dtype=torch.float32, device="cuda")
        plan.run_band(50, 110, [d], 40, 120, [band])
        torch.cuda.synchronize()
        assert torch.equal(band, outs[0][50:110])
        n += 2
        # kf_run_batch: frames overlapping through programmatic dependent launch
        for spec, kind in ((P.harris(300, 200), "b200"), (P.deep10(67, 41), "b200"), (P.harris(64, 48), "unfused")):
            plan, ins, outs = run(spec, kind)
            shape, dt = outs[0].shape, outs[0].dtype
            fin = [[torch.from_numpy(np.ascontiguousarray(ins[0])).cuda()] for _ in range(3)]
            fout = [[torch.empty(shape, dtype=dt, device="cuda")] for _ in range(3)]
            plan.run_batch(fin, fout)
            torch.cuda.synchronize()
            for f in fout:
                assert torch.equal(f[0], outs[0]), spec["name"]
            n += 1
    if which in ("all", "random"):
        for seed in range(10):
            rng = random.Random(70000 + seed)
            dtype = rng.choice(["f32", "u8x4"])
            W, H = rng.choice([(33, 17), (70, 45), (129, 20)])
            spec = P.random_pipeline(rng, W, H, dtype, rng.randint(2, 6))
            for kind in ("unfused", "paper", "b200"):
                run(spec, kind, seed=seed)
                n += 1
    if which in ("all", "peer"):
        # the peer-halo kernels (kf_peer_signal / _pull / _wait) in ONE process: two
        # row bands of a two-input image on this GPU, band 1 pulling band 0's last
        # R rows of both inputs (any alignment: W = 130 is not a multiple of 4)
        W, R = 130, 3
        a = [torch.arange(20 * W, dtype=torch.float32, device="cuda").reshape(20, W) + 1000 * k for k in range(2)]
        b = [torch.full((20 + R, W), -1.0, device="cuda") for _ in range(2)]
        ctr_a = torch.zeros(8, dtype=torch.int32, device="cuda")
        ctr_b = torch.zeros(8, dtype=torch.int32, device="cuda")
        c = lambda t, i: t.data_ptr() + 4 * i   # noqa: E731
        for step in range(3):
            K.peer_signal([c(ctr_b, 0)], c(ctr_a, 6))
            K.peer_pull([x.data_ptr() for x in b], [x.data_ptr() + (20 - R) * W * 4 for x in a], [R * W * 4] * 2,
                        [c(ctr_b, 0)], [c(ctr_b, 2)], [c(ctr_a, 5)], c(ctr_b, 7), 1 << 20, copies=2)
            K.peer_wait([c(ctr_a, 5)], [c(ctr_a, 6)], c(ctr_a, 7), 1 << 20)
        torch.cuda.synchronize()
        for k in range(2):
            assert torch.equal(b[k][:R], a[k][20 - R:]), "peer pull"
        assert int(ctr_a[7]) == 0 and int(ctr_b[7]) == 0 and int(ctr_b[2]) == 3
        n += 3
    print(f"sanitize cases ok: {n} runs")


if __name__ == "__main__":
    main()

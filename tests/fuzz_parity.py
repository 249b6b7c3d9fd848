"""TEST INFRASTRUCTURE (not collected by pytest): a long randomized parity run on
the GPU -- random DAGs (both dtypes, every border mode, radius up to 4,
asymmetric masks, widths from 1 to 2100), random plans (unfused, paper, B200,
ROOFLINE, a random legal partition) and random schedule options, each result
against the oracle (u8x4 bit-exact; f32 normalised <= 1e-5 and pointwise <=
1e-3 on |o| >= 1e-3 max|o|; an output that cancels exactly -- max|o| < 1e-6 for
terms of O(1), e.g. a zero-sum mask on a 1-pixel-wide image -- is rounding noise
on both sides and is compared absolutely, <= 1e-6).  Kernels are compiled up
front in parallel.

    python tests/fuzz_parity.py [n_dags] [seed0] [oracle|bands]   -> one JSON line, exit 1 on any mismatch

Mode `bands` checks the decompositions instead: kf_run_host, random row
bands (kf_run_band) and three kf_run_batch frames against the whole-image
kf_run, bit for bit.
"""
import json
import os
import random
import sys
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from kf_inputs import gen  # noqa: E402
from kf_inputs import pipelines as P  # noqa: E402
from oracle import oracle as O  # noqa: E402
from paper_conf_cgo_qiaorht19_b200 import kfuse as K  # noqa: E402

OPTIONS = [{}, {}, {}, {"tma": 1}, {"rtrip": 2}, {"cta_warps": 4}, {"code_budget": 1000}, {"peel_warmup": 0},
           {"lds_pf": 0}, {"qptr": 0}, {"sring": 0}, {"swring": 0}, {"smem_rows": 6}, {"heavy_first": 0},
           # rolled bodies (small code budget): separate warm-up loop, shared-memory LUT and delay lines, and their
           # alternatives; programmatic dependent launch
           {"code_budget": 1000}, {"code_budget": 1000}, {"code_budget": 1000, "warm_skip": 1},
           {"code_budget": 1000, "warm_skip": 0}, {"code_budget": 1000, "delay_smem": 0},
           {"code_budget": 1000, "lut_smem": 0}, {"pdl": 1}]


def case(i, seed0):
    rng = random.Random(seed0 + i)
    dtype = rng.choice(["f32", "u8x4"])
    W = rng.choice([1, 3, 7, 16, 33, 64, 130, 257, 512, 516, 1024, 2100])
    H = rng.choice([1, 2, 5, 17, 40, 97, 160, 300])
    spec = P.random_pipeline(rng, W, H, dtype, rng.randint(1, 7), max_radius=rng.choice([1, 2, 3, 4]),
                             asym=rng.choice([0.0, 0.3]))
    kind = rng.choice(["unfused", "paper", "b200", "b200roof", "random"])
    opts = rng.choice(OPTIONS)
    lab = None
    if kind == "random":
        n = len(spec["ops"])
        lab = list(range(n))
        edges = sorted({(img - spec["n_inputs"], k) for k, o in enumerate(spec["ops"])
                        for img in o["inputs"] if img >= spec["n_inputs"]})
        rng.shuffle(edges)
        for ks, kd in edges[:rng.randint(0, len(edges))]:
            a, b = lab[ks], lab[kd]
            trial = [a if x == b else x for x in lab]
            try:
                K.Pipeline.from_spec(spec).plan_from_blocks(trial)
                lab = trial
            except K.KfError:
                pass
    return spec, kind, opts, lab, seed0 + i


def make(spec, kind, opts, lab):
    p = K.Pipeline.from_spec(spec, opts)
    if kind == "unfused":
        return p.plan_unfused()
    if kind == "random":
        return p.plan_from_blocks(lab)
    return p.plan_fusion(kind)


def bands_mode(cases):
    """Decompositions: every case again as random row bands (kf_run_band from the
    band's own input rows + halo) and through kf_run_host; both must equal the
    whole-image kf_run bit for bit (REPEAT plans: run_host only)."""
    bad = []
    for spec, kind, opts, lab, seed in cases:
        H, W = spec["height"], spec["width"]
        ins = [gen.image(spec["dtype"], seed + 7 * j, W, H) for j in range(spec["n_inputs"])]
        plan = make(spec, kind, opts, lab)
        d_in = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in ins]
        shape = (H, W) + (() if spec["dtype"] == "f32" else (4,))
        dt = torch.float32 if spec["dtype"] == "f32" else torch.uint8
        full = [torch.empty(shape, dtype=dt, device="cuda") for _ in spec["outputs"]]
        plan.run(d_in, full)
        torch.cuda.synchronize()
        full = [f.cpu().numpy() for f in full]
        host = [np.empty_like(f) for f in full]
        plan.run_host([np.ascontiguousarray(a) for a in ins], host)
        ok = all(np.array_equal(a, b) for a, b in zip(host, full))
        repeat = any(o["kind"] == "local" and o["mode"] == "repeat" for o in spec["ops"])
        if ok and not repeat and H >= 2:
            rng = random.Random(seed)
            cuts = sorted({0, H} | {rng.randint(1, H - 1) for _ in range(rng.randint(1, 4))})
            R = plan.halo_rows
            for r0, r1 in zip(cuts[:-1], cuts[1:]):
                a0, a1 = max(0, r0 - R), min(H, r1 + R)
                b_in = [torch.from_numpy(np.ascontiguousarray(x[a0:a1])).cuda() for x in ins]
                b_out = [torch.empty((r1 - r0,) + shape[1:], dtype=dt, device="cuda") for _ in spec["outputs"]]
                plan.run_band(r0, r1, b_in, a0, a1, b_out)
                torch.cuda.synchronize()
                ok &= all(np.array_equal(o.cpu().numpy(), f[r0:r1]) for o, f in zip(b_out, full))
        if ok:   # three independent frames through kf_run_batch (overlapping launches when single-block)
            fin = [[torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in ins] for _ in range(3)]
            fout = [[torch.empty(shape, dtype=dt, device="cuda") for _ in spec["outputs"]] for _ in range(3)]
            plan.run_batch(fin, fout)
            torch.cuda.synchronize()
            ok &= all(np.array_equal(o.cpu().numpy(), f) for fo in fout for o, f in zip(fo, full))
        if not ok:
            bad.append({"seed": seed, "kind": kind, "opts": opts, "size": [W, H], "dtype": spec["dtype"]})
    return bad


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 200
    seed0 = int(sys.argv[2]) if len(sys.argv) > 2 else 424242
    mode = sys.argv[3] if len(sys.argv) > 3 else "oracle"
    cases = [case(i, seed0) for i in range(n)]
    with ThreadPoolExecutor(max(1, min(32, os.cpu_count() or 1))) as ex:
        list(ex.map(lambda c: make(*c[:4]).compile(), cases))
    if mode == "bands":
        bad = bands_mode(cases)
        print(json.dumps({"mode": "bands", "dags": n, "seed0": seed0, "mismatches": len(bad), "bad": bad[:20]}))
        sys.exit(1 if bad else 0)
    bad, worst, cancelled, ill = [], 0.0, [], []
    for spec, kind, opts, lab, seed in cases:
        ins = [gen.image(spec["dtype"], seed + 7 * j, spec["width"], spec["height"]) for j in range(spec["n_inputs"])]
        plan = make(spec, kind, opts, lab)
        d_in = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in ins]
        shape = (spec["height"], spec["width"]) + (() if spec["dtype"] == "f32" else (4,))
        dt = torch.float32 if spec["dtype"] == "f32" else torch.uint8
        outs = [torch.empty(shape, dtype=dt, device="cuda") for _ in spec["outputs"]]
        plan.run(d_in, outs)
        torch.cuda.synchronize()
        ref = O.run(spec, ins)
        for o, img in zip(outs, spec["outputs"]):
            g, r = o.cpu().numpy(), ref[img]
            err = pw = None
            if spec["dtype"] == "u8x4":
                ok = bool(np.array_equal(g, r))
            else:
                a = np.abs(r)
                d = np.abs(g.astype(np.float64) - r)
                if a.max() < 1e-6:
                    # exact cancellation (e.g. a zero-sum mask on a 1-pixel-wide
                    # image): the fp64 oracle and the f32 kernel both return
                    # rounding noise of O(1) terms; compare absolutely
                    ok = bool(d.max() <= 1e-6)
                    cancelled.append(seed)
                else:
                    err = float(d.max() / a.max())
                    sel = a >= 1e-3 * a.max()
                    pw = float((d[sel] / a[sel]).max())
                    worst = max(worst, err)
                    ok = err <= 1e-5 and pw <= 1e-3
            if not ok and spec["dtype"] == "f32" and kind == "unfused" and err is not None and err <= 1e-5:
                # the unfused plan IS the f32 reference execution (one kernel per
                # operator): a pointwise miss within the normalised bound is f32
                # conditioning of the random program
                ill.append({"seed": seed, "unfused_pw": pw, "unfused_norm": err})
                ok = True
            if not ok and spec["dtype"] == "f32" and kind != "unfused":
                # f32 conditioning, not fusion: a random program (cancelling
                # differences, ABS near zero) can exceed the pointwise bound in
                # plain f32.  If the unfused GPU plan -- one kernel per operator,
                # every intermediate materialised in f32 -- misses the oracle by as
                # much, the fused result is as exact as f32 execution allows.
                u = make(spec, "unfused", {}, None)
                uo = [torch.empty(shape, dtype=dt, device="cuda") for _ in spec["outputs"]]
                u.run(d_in, uo)
                torch.cuda.synchronize()
                ug = uo[spec["outputs"].index(img)].cpu().numpy()
                ud = np.abs(ug.astype(np.float64) - r)
                a = np.abs(r)
                sel = a >= 1e-3 * a.max()
                upw = float((ud[sel] / a[sel]).max()) if a.max() >= 1e-6 else 0.0
                fpw = float((d[sel] / a[sel]).max()) if a.max() >= 1e-6 else 0.0
                uerr = float(ud.max() / max(a.max(), 1e-30))
                if upw > 1e-3 and fpw <= 4 * upw and float(d.max()) <= 4 * float(ud.max()) + 1e-12:
                    ill.append({"seed": seed, "fused_pw": fpw, "unfused_pw": upw, "unfused_norm": uerr})
                    ok = True
            if not ok:
                bad.append({"seed": seed, "kind": kind, "opts": opts, "size": [spec["width"], spec["height"]],
                            "dtype": spec["dtype"], "ops": len(spec["ops"])})
    print(json.dumps({"dags": n, "seed0": seed0, "mismatches": len(bad), "worst_norm_err_f32": worst,
                      "cancelled_outputs": len(cancelled), "ill_conditioned_in_f32": ill[:20], "bad": bad[:20]}))
    sys.exit(1 if bad else 0)


if __name__ == "__main__":
    main()

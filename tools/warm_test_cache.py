"""Pre-compiles (NVRTC, no GPU needed) the fused kernels the GPU test suite and
the bench will launch, into the in-tree cubin cache (paper_conf_cgo_qiaorht19_b200/
kcache/, keyed by source hash), so that a fresh GPU box only loads modules.
Runs the compiles in parallel processes.  Scratch tooling, not the product.

    python tools/warm_test_cache.py [-j N]
"""
import argparse
import os
import random
import sys
from multiprocessing import Pool

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def jobs():
    from kf_inputs import pipelines as P
    out = []   # (spec, kind, options, hooks)
    for wl in ["harris", "shitomasi", "unsharp", "sobel", "enhance", "deep10"]:
        for size in [(67, 41), (256, 256)]:
            for kind in ("unfused", "paper", "b200"):
                out.append((P.WORKLOADS[wl](*size), kind, None, False))
    for wl in ["harris", "deep10"]:
        for mode in P.MODES:
            out.append((P.WORKLOADS[wl](45, 37, mode=mode), "b200", None, False))
    for size in [(1, 1), (2, 3), (3, 2), (5, 5), (31, 9), (33, 17), (7, 70)]:
        for wl in ["harris", "deep10", "unsharp"]:
            for mode in P.MODES:
                out.append((P.WORKLOADS[wl](*size, mode=mode), "b200", None, False))
    for seed in range(60):
        rng = random.Random(70000 + seed)
        dtype = rng.choice(["f32", "u8x4"])
        W, H = rng.choice([(1, 1), (4, 3), (9, 9), (33, 17), (70, 45), (129, 20)])
        spec = P.random_pipeline(rng, W, H, dtype, rng.randint(2, 8))
        for kind in ("unfused", "paper", "b200"):
            out.append((spec, kind, None, False))
    for seed in range(40):
        rng = random.Random(91000 + seed)
        dtype = rng.choice(["f32", "u8x4"])
        W, H = rng.choice([(512, 70), (516, 33), (1024, 41), (640, 131), (2048, 24), (513, 37)])
        spec = P.random_pipeline(rng, W, H, dtype, rng.randint(2, 6), max_radius=4, asym=0.4)
        for kind in ("unfused", "paper", "b200"):
            out.append((spec, kind, None, False))
    for cfg in ["C1", "C2", "C3", "C3s", "C4", "C5"]:
        spec, _ = P.config(cfg)
        for kind in ("unfused", "paper", "b200", "basic"):
            out.append((spec, kind, None, False))
    for wl in ["sobel", "enhance"]:
        for kind in ("unfused", "paper", "b200", "basic"):
            out.append((P.WORKLOADS[wl](2048, 2048), kind, None, False))
    same = [{"qptr": 0}, {"lds_pf": 0}, {"const_w": 0}, {"heavy_first": 0}, {"pro_rp": 0}, {"smem_rows": 6},
            {"sring": 0}, {"minctas": 8}, {"code_budget": 1000}, {"swring": 0}, {"tma": 1},
            {"tma": 1, "lds_pf": 0}, {"tma": 1, "code_budget": 1000}, {"tma": 1, "smem_rows": 6}, {"rtrip": 2},
            {"rtrip": 2, "code_budget": 1000}, {"code_budget": 1000, "lds_pf": 0}, {"cta_warps": 2},
            {"cta_warps": 4}, {"cta_warps": 8}, {"cta_warps": 4, "tma": 1}, {"cta_warps": 4, "code_budget": 1000},
            {"peel_warmup": 0}, {"peel_warmup": 0, "lds_pf": 0}, {"pdl": 1},
            {"warm_skip": 0}, {"warm_skip": 0, "code_budget": 1000}, {"warm_skip": 1},
            {"warm_skip": 1, "code_budget": 1000}, {"pdl": 1, "code_budget": 1000}, {"lut_smem": 0},
            {"delay_smem": 0}, {"delay_smem": 1, "code_budget": 1000}, {"pdl": 0}]
    exp = [{"v8": 1}, {"persist": 1}, {"nlong": 3}]
    for wl in ["harris", "unsharp", "shitomasi"]:
        for o in ({"pairs": 0}, {"defer": 0}):
            out.append((P.WORKLOADS[wl](200, 150), "b200", o, True))
    for cfg in ["C2", "C3", "C3s", "C4"]:
        spec, _ = P.config(cfg)
        out.append((spec, "b200", {"tma": 1}, False))
    out.append((P.copy(4096, 4096), "b200", {"tma": 1}, False))
    out.append((P.copy(4096, 4096), "b200", None, False))
    for o in ({"peel_warmup": 0},):
        for cfg in ("C2", "C3", "C3s", "C4", "C5"):
            out.append((P.config(cfg)[0], "b200", o, False))
        out.append((P.copy(4096, 4096), "b200", o, False))
    out.append((P.config("C4")[0], "b200", {"rtrip": 2}, False))
    out.append((P.enhance(2048, 2048), "b200", {"rtrip": 2}, False))
    for wl in ["harris", "deep10", "unsharp"]:
        for o in same:
            out.append((P.WORKLOADS[wl](200, 150), "b200", o, False))
        for o in exp:
            out.append((P.WORKLOADS[wl](200, 150), "b200", o, True))
    for mode in ("clamp", "constant"):
        out.append((P.fig4(mode), "whole", {"naive_border": 1}, True))
        out.append((P.harris(8, 8, mode), "whole", {"naive_border": 1}, True))
        out.append((P.fig4(mode), "whole", None, False))
        out.append((P.harris(8, 8, mode), "whole", None, False))
    for wl in ["harris", "deep10", "two_input"]:
        out.append((P.WORKLOADS[wl](96, 130), "b200", None, False))
        out.append((P.WORKLOADS[wl](130, 130), "b200", None, False))
    for wl in ["harris", "deep10", "unsharp"]:
        for kind in ("unfused", "paper", "b200"):
            out.append((P.WORKLOADS[wl](130, 1030), kind, None, False))
    for wl in ["harris", "deep10"]:
        out.append((P.WORKLOADS[wl](300, 200), "b200", None, False))
    out.append((P.harris(512, 384), "b200", None, False))     # examples/harris_c.c
    for o in ({"host_bands": 1}, {"host_bands": 3}, {"host_bands": 16}, {"host_bands": 32},
              {"host_bands": 12, "host_taper": 0}, {"host_direct": 1}):
        out.append((P.harris(130, 1030), "b200", o, False))
    for width in (130, 128, 516):   # test_swar_constant_border_below_producer_range
        p = P.Pipeline("constant_edge", width, 17, "u8x4")
        i = p.input()
        a = p.point("p3", [i], [P.L(0), P.C(3), P.MUL, P.SHR(2), P.SAT])
        b = p.point("p4", [a, i], [P.L(0), P.L(1), P.ADD, P.C(128), P.ADD, P.SAT])
        p.output(p.local("l5", b, [[16, -8, 8]], "constant", constant=0.0,
                         post=[P.L(0), P.C(16), P.ADD, P.SHR(5), P.C(0), P.ADD, P.SAT]))
        for o in (None, {"code_budget": 1000}):
            out.append((p.spec(), "b200", o, False))
    for dtype in ("f32", "u8x4"):   # test_two_constant_borders_on_one_row
        for width in (512, 130):
            p = P.Pipeline("two_constants", width, 64, dtype)
            i = p.input()
            mix = [[1, 0, 2], [0, 1, 0], [3, 0, 1]]
            if dtype == "f32":
                a = p.local("a", i, [[0.25, 0.5, 0.25]], "mirror101")
                b = p.local("b", a, [[v / 8.0 for v in r] for r in mix], "constant", constant=0.0)
                c = p.local("c", a, [[v / 8.0 for v in r] for r in mix], "constant", constant=1.0)
                p.output(p.point("d", [b, c], [P.L(0), P.L(1), P.SUB]))
            else:
                a = p.local("a", i, [[1, 2, 1]], "mirror101", post=[P.L(0), P.C(2), P.ADD, P.SHR(2), P.SAT])
                b = p.local("b", a, mix, "constant", constant=0.0, post=[P.L(0), P.SHR(3), P.SAT])
                c = p.local("c", a, mix, "constant", constant=255.0, post=[P.L(0), P.SHR(3), P.SAT])
                p.output(p.point("d", [b, c], [P.L(0), P.L(1), P.SUB, P.C(255), P.ADD, P.SHR(1), P.SAT]))
            out.append((p.spec(), "whole", None, False))
    out.append((P.deep10(260, 150), "b200", None, False))
    out.append((P.two_input(512, 300), "b200", None, False))
    out.append((P.harris(130, 97), "b200", None, False))
    out.append((P.harris(130, 1030), "unfused", None, False))
    for mode in P.MODES:
        for size in [(128, 96), (516, 70)]:
            out.append((P.deep10(*size, mode=mode), "b200", None, False))
            out.append((P.swar_stress(*size, mode=mode), "b200", None, False))
    # the bounds-checking build's launches (tests/test_bounds.py)
    import importlib.util
    bspec = importlib.util.spec_from_file_location("bounds_cases", os.path.join(ROOT, "tests", "bounds_cases.py"))
    bc = importlib.util.module_from_spec(bspec)
    bspec.loader.exec_module(bc)
    for _, spec, kind, o in bc.cases():
        out.append((spec, kind, o, "bounds"))
        out.append((spec, kind, o, False))   # the product twin each bounds-checked result is compared with
    out.append((P.harris(300, 200), "b200", {"bounds_shrink": 1}, "bounds"))
    for wl in ["harris", "deep10"]:
        out.append((P.WORKLOADS[wl](300, 200), "b200", None, "bounds"))
        out.append((P.WORKLOADS[wl](130, 1030), "b200", None, "bounds"))
    return out


_MODS = {}


def _mod(hooks):
    """The product binding (hooks False), the test-hooks build (True) or the
    bounds-checking build ("bounds")."""
    from paper_conf_cgo_qiaorht19_b200 import kfuse as K
    if not hooks:
        return K
    name = "libkfuse_bounds.so" if hooks == "bounds" else "libkfuse_testhooks.so"
    if name not in _MODS:
        import importlib.util
        spec = importlib.util.spec_from_file_location("kfuse_" + name.split(".")[0], K.__file__)
        m = importlib.util.module_from_spec(spec)
        spec.loader.exec_module(m)
        m.lib = m._open(os.path.join(os.path.dirname(K.__file__), name))
        _MODS[name] = m
    return _MODS[name]


def compile_job(job):
    spec, kind, opts, hooks = job
    K = _mod(hooks)
    try:
        p = K.Pipeline.from_spec(spec, opts)
        plan = (p.plan_unfused() if kind == "unfused" else p.plan_from_blocks([0] * len(spec["ops"]))
                if kind == "whole" else p.plan_basic("paper") if kind == "basic" else p.plan_fusion(kind))
        plan.compile()
        return None
    except Exception as e:   # noqa: BLE001
        return f"{spec['name']} {spec['width']}x{spec['height']} {kind} {opts}: {str(e)[:300]}"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("-j", type=int, default=os.cpu_count())
    ap.add_argument("--prune", action="store_true", help="delete cached cubins this warm-up did not use")
    a = ap.parse_args()
    import time
    t0 = time.time() - 2
    js = jobs()
    with Pool(a.j) as pool:
        errs = [e for e in pool.imap_unordered(compile_job, js, chunksize=1) if e]
    print(f"{len(js)} plans compiled, {len(errs)} failures")
    if a.prune and not errs:
        cache = os.path.join(ROOT, "paper_conf_cgo_qiaorht19_b200", "kcache")
        old = [f for f in os.listdir(cache) if os.path.getmtime(os.path.join(cache, f)) < t0]
        for f in old:
            os.remove(os.path.join(cache, f))
        print(f"pruned {len(old)} unused cubins")
    for e in errs:
        print("FAIL", e)
    sys.exit(1 if errs else 0)


if __name__ == "__main__":
    main()

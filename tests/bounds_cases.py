"""TEST INFRASTRUCTURE (not collected by pytest): the launches the bounds-checking
build (libkfuse_bounds.so, KF_BOUNDS) is run on by tests/test_bounds.py -- every
plan kind, every border mode, tiny / ragged / W % 4 != 0 images, the schedule
options that change the memory path (TMA feed, several warps per CTA, rolled
bodies, smaller rings, no smem ring), random DAGs, and the full-size bench
configurations.  Listed here so that tools/warm_test_cache.py can pre-compile
the same kernels."""
import random

from kf_inputs import pipelines as P


def cases():
    out = []   # (id, spec, plan kind, options)
    for wl in ["harris", "shitomasi", "unsharp", "sobel", "enhance", "deep10", "two_input"]:
        for size in [(67, 41), (256, 240), (130, 97)]:
            for kind in ("unfused", "paper", "b200"):
                out.append((f"{wl}-{size[0]}x{size[1]}-{kind}", P.WORKLOADS[wl](*size), kind, None))
    for wl in ["harris", "deep10", "unsharp"]:
        for mode in P.MODES:
            for size in [(45, 37), (5, 5), (33, 17)]:
                out.append((f"{wl}-{mode}-{size[0]}x{size[1]}", P.WORKLOADS[wl](*size, mode=mode), "b200", None))
    for o in ({"tma": 1}, {"cta_warps": 4}, {"code_budget": 1000}, {"smem_rows": 6}, {"sring": 0},
              {"peel_warmup": 0}, {"rtrip": 2, "code_budget": 1000}, {"warm_skip": 0}, {"warm_skip": 1},
              {"delay_smem": 0}, {"code_budget": 1000, "warm_skip": 1}):
        tag = ",".join(f"{k}={v}" for k, v in o.items())
        for wl in ["harris", "deep10", "unsharp"]:
            out.append((f"{wl}-200x150-{tag}", P.WORKLOADS[wl](200, 150), "b200", o))
    for seed in range(12):
        rng = random.Random(93000 + seed)
        dtype = rng.choice(["f32", "u8x4"])
        W, H = rng.choice([(33, 17), (70, 45), (129, 20), (516, 33), (513, 37)])
        spec = P.random_pipeline(rng, W, H, dtype, rng.randint(2, 6), max_radius=4, asym=0.4)
        for kind in ("unfused", "b200"):
            out.append((f"random{seed}-{kind}", spec, kind, None))
    for cfg in ["C2", "C3", "C4"]:
        out.append((f"{cfg}-full", P.config(cfg)[0], "b200", None))
    return out

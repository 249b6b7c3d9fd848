"""Host-side memory/UB check (no GPU): drives the planners, the exact planner and
the code generator of an ASan+UBSan build of libkfuse (tools/asan_host.sh) over
150 random DAGs x 3 profiles x 3 planners and every workload under several
schedule options.  Diagnostics only."""
import os, sys, random
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cgo_qiaorht19_b200 import kfuse as K
K.lib = K._open(os.environ.get("KF_ASAN_LIB", "/tmp/kf_asan/libkfuse.so"))
from kf_inputs import pipelines as P
n = 0
for seed in range(150):
    rng = random.Random(555 + seed)
    dtype = rng.choice(["f32", "u8x4"])
    W, H = rng.choice([(16, 12), (70, 45), (513, 37), (2048, 24), (1, 1), (5, 3)])
    spec = P.random_pipeline(rng, W, H, dtype, rng.randint(1, 8), max_radius=rng.choice([2, 4]), asym=0.3)
    for prof in ("paper", "b200", "b200roof"):
        p = K.Pipeline.from_spec(spec)
        for plan in (p.plan_fusion(prof), p.plan_basic(prof), p.plan_unfused()):
            for b in range(plan.num_launches):
                plan.source(b)
            _ = plan.blocks, plan.objective, plan.cuts, plan.halo_rows
            n += 1
        if len(spec["ops"]) <= 10:
            K.Pipeline.from_spec(spec).plan_exact(prof)
for wl in ("harris", "shitomasi", "unsharp", "sobel", "enhance", "deep10", "two_input"):
    spec = P.WORKLOADS[wl](300, 200)
    for opts in ({}, {"tma": 1}, {"cta_warps": 4}, {"rtrip": 2}, {"code_budget": 1000}, {"peel_warmup": 0}):
        plan = K.Pipeline.from_spec(spec, opts).plan_fusion("b200")
        plan.source(0)
        n += 1
print("asan drive ok", n)

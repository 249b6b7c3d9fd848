"""B200 calibration of the fusion benefit model and the Table I shape on B200
(SURVEY §8(f)1 and §8(f)2).  Runs on the GPU box:

    python tools/calibrate.py [--size 2048] [--samples 14] [--out gpurun_out/calibration.json]

1. Hardware-model constants (Eqs. 3-7: tg, ts, cALU, cSFU)
   measured by tools/ubench/model_consts.cu on this B200 -> the "b200cal"
   profile: the measured latencies, the staged recompute factor phi of the
   B200 profile (R-4) with the streaming kernel's tile -- a 120-pixel column
   chunk by a 32-row strip -- and cMshared = 5.
2. For every paper application (Harris, ShiTomasi, Unsharp, Sobel, Enhance, and
   the deep10 C4 body) at the paper's 2048x2048 size: the named plans (unfused,
   basic [12], Alg. 1 under the paper / B200 / b200cal / b200roof profiles, the
   exact optimum under b200cal and b200roof) plus random executable partitions (random merges along
   edges accepted by kf_plan_from_blocks).  Each plan's objective beta (Eq. 1:
   the sum of the b200cal weights of the edges inside blocks; eps edges count 0
   with their number reported) is set against its measured time (CUDA-graph
   replay, 4 rotating buffer sets).  Spearman's rank correlation between beta
   and time says whether the calibrated model ranks plans the way B200 does --
   for the b200cal weights (the paper's Eqs. 3-12 with measured latencies) and
   for the ROOFLINE weights (R-20: per-pair max(DRAM time, issue
   time), the issue-rate extension for compute-bound blocks).
3. Table I shape: speedups of basic and optimized fusion over unfused, and of
   optimized over basic, per application.

Diagnostics only: no product code path reads its output.
"""
from __future__ import annotations

import argparse
import json
import os
import random
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from kf_inputs import gen  # noqa: E402
from kf_inputs import pipelines as P  # noqa: E402
from paper_conf_cgo_qiaorht19_b200 import kfuse as K  # noqa: E402

APPS = ["harris", "shitomasi", "unsharp", "sobel", "enhance", "deep10"]


def measure_consts() -> dict:
    src = os.path.join(ROOT, "tools", "ubench", "model_consts.cu")
    exe = os.path.join(ROOT, "tools", "ubench", "model_consts")
    subprocess.run(["nvcc", "-O3", "-gencode", "arch=compute_100a,code=sm_100a", "-o", exe, src], check=True)
    out = subprocess.run([exe], capture_output=True, text=True, check=True).stdout
    return json.loads(out.strip().splitlines()[-1])


def cal_params(c: dict) -> K.ModelParams:
    return K.model_params("b200", tg=c["tg"], ts=c["ts"], c_alu=c["c_alu"], c_sfu=c["c_sfu"],
                          tile_w=120, tile_h=32)


def time_plan(plan, ins, outs, steps=60) -> float:
    plan.prepare()
    s = torch.cuda.Stream()
    n = len(ins)
    for i in range(5):
        plan.run([ins[i % n]], [outs[i % n]], s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for i in range(steps):
            plan.run([ins[i % n]], [outs[i % n]], s)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        g.replay()
        torch.cuda.synchronize()
        e0.record(s)
        g.replay()
        e1.record(s)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / steps * 1e3   # us


def beta(blocks, weights) -> tuple[float, int]:
    b, ne = 0.0, 0
    for blk in blocks:
        S = set(blk)
        for (ks, kd), e in weights.items():
            if ks in S and kd in S:
                if e["is_eps"]:
                    ne += 1
                else:
                    b += e["w"]
    return b, ne


def random_partitions(spec, rng, n_samples, tries=400) -> list:
    n = len(spec["ops"])
    edges = sorted({(img - spec["n_inputs"], k) for k, o in enumerate(spec["ops"])
                    for img in o["inputs"] if img >= spec["n_inputs"]})
    seen, out = set(), []
    for _ in range(tries):
        lab = list(range(n))
        order = edges[:]
        rng.shuffle(order)
        stop = rng.randint(0, len(order))
        for ks, kd in order[:stop]:
            a, b = lab[ks], lab[kd]
            if a == b:
                continue
            trial = [a if x == b else x for x in lab]
            try:
                K.Pipeline.from_spec(spec).plan_from_blocks(trial)
            except K.KfError:
                continue
            lab = trial
        key = tuple(sorted(tuple(sorted(k for k in range(n) if lab[k] == L)) for L in set(lab)))
        if key not in seen:
            seen.add(key)
            out.append(lab)
        if len(out) >= n_samples:
            break
    return out


def t_of(rows, name):
    return next(r["us"] for r in rows if r["plan"] == name)


def spearman(x, y) -> float:
    def ranks(v):
        order = sorted(range(len(v)), key=lambda i: v[i])
        r = [0.0] * len(v)
        i = 0
        while i < len(order):
            j = i
            while j + 1 < len(order) and v[order[j + 1]] == v[order[i]]:
                j += 1
            for t in range(i, j + 1):
                r[order[t]] = (i + j) / 2.0
            i = j + 1
        return r
    rx, ry = ranks(x), ranks(y)
    n = len(x)
    mx, my = sum(rx) / n, sum(ry) / n
    cov = sum((a - mx) * (b - my) for a, b in zip(rx, ry))
    vx = sum((a - mx) ** 2 for a in rx) ** 0.5
    vy = sum((b - my) ** 2 for b in ry) ** 0.5
    return cov / (vx * vy) if vx > 0 and vy > 0 else float("nan")


def _compile_labels(job):
    app, size, lab = job
    spec = P.WORKLOADS[app](size, size)
    K.Pipeline.from_spec(spec).plan_from_blocks(lab).compile()


def compile_only(size: int, samples: int) -> None:
    """Warms the in-tree cubin cache with every plan main() will time (no GPU)."""
    from multiprocessing import Pool
    rng = random.Random(2019)
    jobs = []
    for app in APPS:
        spec = P.WORKLOADS[app](size, size)
        p = K.Pipeline.from_spec(spec)
        for plan in (p.plan_unfused(), p.plan_basic("paper"), p.plan_fusion("paper"), p.plan_fusion("b200"),
                     p.plan_fusion("b200roof"), p.plan_exact("b200roof")):
            lab = [0] * len(spec["ops"])
            for bi, ks in enumerate(plan.blocks):
                for k in ks:
                    lab[k] = bi
            jobs.append((app, size, lab))
        jobs += [(app, size, lab) for lab in random_partitions(spec, rng, samples)]
    with Pool(os.cpu_count()) as pool:
        pool.map(_compile_labels, jobs, chunksize=1)
    print(f"compiled {len(jobs)} plans")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--compile-only", action="store_true")
    ap.add_argument("--size", type=int, default=2048)
    ap.add_argument("--samples", type=int, default=24)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "calibration.json"))
    a = ap.parse_args()
    if a.compile_only:
        compile_only(a.size, a.samples)
        return
    consts = measure_consts()
    mcal = cal_params(consts)
    print(json.dumps({"consts": consts}), flush=True)
    rng = random.Random(2019)
    report = {"consts": consts, "profile_b200cal": {f: getattr(mcal, f) for f, _ in K.ModelParams._fields_},
              "size": a.size, "apps": {}}
    for app in APPS:
        spec = P.WORKLOADS[app](a.size, a.size)
        W = H = a.size
        host = gen.image(spec["dtype"], 7, W, H)
        tdt = torch.float32 if spec["dtype"] == "f32" else torch.uint8
        oshape = (H, W) if spec["dtype"] == "f32" else (H, W, 4)
        ins = [torch.from_numpy(host).cuda() for _ in range(4)]
        outs = [torch.empty(oshape, dtype=tdt, device="cuda") for _ in range(4)]
        def edge_table(prof):
            ref = K.Pipeline.from_spec(spec).plan_fusion(prof)
            wt = {}
            for k, o in enumerate(spec["ops"]):
                for img in o["inputs"]:
                    if img >= spec["n_inputs"]:
                        wt[(img - spec["n_inputs"], k)] = ref.edge(img - spec["n_inputs"], k)
            return wt
        weights = edge_table(mcal)
        weights_roof = edge_table(K.model_params("b200roof"))
        named = {
            "unfused": lambda p: p.plan_unfused(),
            "basic": lambda p: p.plan_basic("paper"),
            "alg1_paper": lambda p: p.plan_fusion("paper"),
            "alg1_b200": lambda p: p.plan_fusion("b200"),
            "alg1_b200cal": lambda p: p.plan_fusion(mcal),
            "exact_b200cal": lambda p: p.plan_exact(mcal),
            "alg1_b200roof": lambda p: p.plan_fusion("b200roof"),
            "exact_b200roof": lambda p: p.plan_exact("b200roof"),
        }
        rows = []
        done = set()
        for name, mk in named.items():
            plan = mk(K.Pipeline.from_spec(spec))
            key = tuple(map(tuple, plan.blocks))
            b, ne = beta(plan.blocks, weights)
            br, _ = beta(plan.blocks, weights_roof)
            us = time_plan(plan, ins, outs)
            rows.append({"plan": name, "blocks": plan.blocks, "beta": round(b, 2), "eps": ne,
                         "beta_roof": round(br, 5), "launches": plan.num_launches, "us": round(us, 2)})
            done.add(key)
        for lab in random_partitions(spec, rng, a.samples):
            plan = K.Pipeline.from_spec(spec).plan_from_blocks(lab)
            key = tuple(map(tuple, plan.blocks))
            if key in done:
                continue
            done.add(key)
            b, ne = beta(plan.blocks, weights)
            br, _ = beta(plan.blocks, weights_roof)
            us = time_plan(plan, ins, outs)
            rows.append({"plan": "random", "blocks": plan.blocks, "beta": round(b, 2), "eps": ne,
                         "beta_roof": round(br, 5), "launches": plan.num_launches, "us": round(us, 2)})
        t = {r["plan"]: r["us"] for r in rows if r["plan"] != "random"}
        rho = spearman([r["beta"] for r in rows], [r["us"] for r in rows])
        rho_roof = spearman([r["beta_roof"] for r in rows], [r["us"] for r in rows])
        best = min(rows, key=lambda r: r["us"])
        d = {"workload": f"{app} {W}x{H} {spec['dtype']}", "plans": rows,
             "spearman_beta_vs_time": round(rho, 3),
             "spearman_beta_roof_vs_time": round(rho_roof, 3),
             "alg1_b200roof_us": t_of(rows, "alg1_b200roof"), "alg1_b200_us": t_of(rows, "alg1_b200"),
             "fastest": best["plan"], "fastest_blocks": best["blocks"],
             "table1": {"basic_over_unfused": round(t["unfused"] / t["basic"], 3),
                        "optimized_paper_over_unfused": round(t["unfused"] / t["alg1_paper"], 3),
                        "optimized_b200_over_unfused": round(t["unfused"] / t["alg1_b200"], 3),
                        "optimized_b200cal_over_unfused": round(t["unfused"] / t["alg1_b200cal"], 3),
                        "optimized_paper_over_basic": round(t["basic"] / t["alg1_paper"], 3),
                        "optimized_b200cal_over_basic": round(t["basic"] / t["alg1_b200cal"], 3)}}
        report["apps"][app] = d
        print(json.dumps({app: {k: v for k, v in d.items() if k != "plans"}}), flush=True)
        del ins, outs
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(report, f, indent=1)


if __name__ == "__main__":
    main()

"""Schedule-option sweep on the GPU box: times one config/plan under several
option settings (kf_set_option; every option keeps the results bit-identical).
Prints one JSON line per setting.  Diagnostics only -- bench.py is the
measurement of record.

    python tools/sweep.py --config C3 --plan b200 '' 'tma=1' 'tma=1 smem_rows=8'
    python tools/sweep.py --config copy:4096:4096 '' 'tma=1'
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def _binding(lib: str):
    """The product binding, or a second instance bound to the test-hooks build
    (experimental options) when lib == 'testhooks'."""
    from paper_conf_cgo_qiaorht19_b200 import kfuse as K
    if lib != "testhooks":
        return K
    import importlib.util
    spec = importlib.util.spec_from_file_location("kfuse_testhooks", K.__file__)
    mod = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mod)
    mod.lib = mod._open(os.path.join(os.path.dirname(K.__file__), "libkfuse_testhooks.so"))
    return mod


def time_setting(cfg: str, plan_kind: str, steps: int, opts: dict, reps: int, lib: str = "product") -> dict:
    import torch
    from kf_inputs import gen
    from kf_inputs import pipelines as P
    K = _binding(lib)
    if ":" in cfg:   # workload:W:H
        wl, w, h = cfg.split(":")
        spec, seed = P.WORKLOADS[wl](int(w), int(h)), 1
    else:
        spec, seed = P.config(cfg)
    W, H = spec["width"], spec["height"]
    host = gen.image(spec["dtype"], seed, W, H)
    nsets = max(2, min(8, int(512e6 // (8 * W * H))))
    ins = [torch.from_numpy(host).cuda() for _ in range(nsets)]
    outs = [torch.empty_like(x) for x in ins]
    p = K.Pipeline.from_spec(spec, opts)
    plan = p.plan_unfused() if plan_kind == "unfused" else p.plan_fusion(plan_kind)
    plan.prepare()
    s = torch.cuda.Stream()
    for i in range(10):
        plan.run([ins[i % nsets]], [outs[i % nsets]], s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for i in range(steps):
            plan.run([ins[i % nsets]], [outs[i % nsets]], s)
    us = []
    with torch.cuda.stream(s):            # replay() launches on the current stream
        g.replay()
        torch.cuda.synchronize()
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            g.replay()
            e1.record(s)
            torch.cuda.synchronize()
            us.append(e0.elapsed_time(e1) / steps * 1e3)
    us.sort()
    med = us[len(us) // 2]
    ref = outs[0].clone()
    del g, ins, outs
    torch.cuda.empty_cache()
    return {"us_median": round(med, 2), "us_min": round(us[0], 2), "gpx_s": round(W * H / med / 1e3, 1),
            "out_sum": float(ref.double().sum().item())}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C3")
    ap.add_argument("--plan", default="b200")
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--reps", type=int, default=7)
    ap.add_argument("--lib", default="product", choices=["product", "testhooks"])
    ap.add_argument("settings", nargs="*")
    a = ap.parse_args()
    for st in a.settings or [""]:
        opts = {}
        for kv in st.split():
            k, v = kv.split("=", 1)
            opts[k] = int(v)
        try:
            r = time_setting(a.config, a.plan, a.steps, opts, a.reps, a.lib)
        except Exception as e:   # noqa: BLE001
            r = {"error": f"{type(e).__name__}: {str(e)[:300]}"}
        print(json.dumps({"config": a.config, "plan": a.plan, "lib": a.lib, "setting": st, **r}), flush=True)


if __name__ == "__main__":
    main()

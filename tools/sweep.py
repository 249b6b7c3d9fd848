"""Tuning sweep on the GPU box: times one config/plan under several env knob
settings (KFUSE_PREFETCH, KFUSE_MINCTAS, KFUSE_DIAG_SKIP), each in its own
subprocess so the code generator sees the knobs.  Prints one JSON line per
setting.  Diagnostics only -- bench.py is the measurement of record.

    python tools/sweep.py --config C3 --plan b200 'KFUSE_PREFETCH=2' 'KFUSE_PREFETCH=6 KFUSE_MINCTAS=20'
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def child(cfg: str, plan_kind: str, steps: int) -> None:
    sys.path.insert(0, ROOT)
    import torch
    from kf_inputs import gen
    from kf_inputs import pipelines as P
    from paper_conf_cgo_qiaorht19_b200 import kfuse as K
    if ":" in cfg:   # workload:W:H
        wl, w, h = cfg.split(":")
        spec, seed = P.WORKLOADS[wl](int(w), int(h)), 1
    else:
        spec, seed = P.config(cfg)
    W, H = spec["width"], spec["height"]
    host = gen.image(spec["dtype"], seed, W, H)
    ins = [torch.from_numpy(host).cuda() for _ in range(4)]
    outs = [torch.empty_like(x) for x in ins]
    p = K.Pipeline.from_spec(spec)
    plan = p.plan_unfused() if plan_kind == "unfused" else p.plan_fusion(plan_kind)
    plan.prepare()
    s = torch.cuda.Stream()
    for i in range(10):
        plan.run([ins[i % 4]], [outs[i % 4]], s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for i in range(steps):
            plan.run([ins[i % 4]], [outs[i % 4]], s)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):            # replay() launches on the current stream
        g.replay()
        torch.cuda.synchronize()
        e0.record(s)
        g.replay()
        e1.record(s)
    torch.cuda.synchronize()
    us = e0.elapsed_time(e1) / steps * 1e3
    print(json.dumps({"us": round(us, 2), "gpx_s": round(W * H / us / 1e3, 1)}))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C3")
    ap.add_argument("--plan", default="b200")
    ap.add_argument("--steps", type=int, default=500)
    ap.add_argument("--child", action="store_true")
    ap.add_argument("settings", nargs="*")
    a = ap.parse_args()
    if a.child:
        child(a.config, a.plan, a.steps)
        return
    for st in a.settings or [""]:
        env = dict(os.environ)
        for kv in st.split():
            k, v = kv.split("=", 1)
            env[k] = v
        r = subprocess.run([sys.executable, __file__, "--child", "--config", a.config, "--plan", a.plan,
                            "--steps", str(a.steps)], env=env, capture_output=True, text=True)
        out = r.stdout.strip().splitlines()[-1] if r.stdout.strip() else r.stderr.strip()[-300:]
        print(json.dumps({"config": a.config, "plan": a.plan, "setting": st, "result": out}), flush=True)


if __name__ == "__main__":
    main()

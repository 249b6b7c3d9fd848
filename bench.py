#!/usr/bin/env python
"""Benchmark of the fused image-pipeline hot path on B200 (BASELINE.json metric:
"Harris 4096^2 Mpixel/s fused vs unfused; DRAM bytes/pixel; HBM GB/s vs peak").

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl kfuse|reference]
                    [--config C3] [--plan b200]

N=1: workload C3 = Harris 4096x4096 float32 (clamp), the B200-profile plan
(fully fused, one launch per step).  A step = one kf_run over one image, inputs
already resident in HBM; 4 rotating input/output buffer sets (512 MiB > the
126 MB L2) so consecutive steps never hit in L2.  Every plan (unfused, basic
[12], paper profile, B200 profile) is timed the same way, and so are the other
BASELINE configs (C1, C2, C3s, C4, C5 at one GPU) and Sobel / Enhance at 2048^2
(the paper's Table I shape) under "workloads".
N>1 (torchrun): the headline is weak scaling by row bands -- each rank a
4096x4096 band of a (4096N)x4096 image -- and "strong_c5" adds BASELINE C5
(one 16384x16384 Harris image, 16384/N rows per GPU).  Every step exchanges
the R halo rows with the neighbours (peer-memory pull over NVLink, or NCCL
send/recv) behind the band's core rows, then computes the edge strips.
--impl reference: the unfused CPU oracle (oracle/) timed on the host cores on
the headline's full image.  One JSON line on stdout (rank 0).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "Harris 4096² Mpixel/s fused vs unfused; DRAM bytes/pixel; HBM GB/s vs peak"
UNIT = "Mpixel/s"
DATA = "synthetic: counter-based SplitMix64 uniform [0,1) images (kf_inputs/gen.py), as the paper's random images"
PLANS = ("unfused", "basic", "paper", "b200")
# the other BASELINE.json configs, timed beside the headline (parity cases otherwise),
# and the paper's Sobel / Enhancement apps at its 2048^2 size (Table I shape)
EXTRA_CONFIGS = ("C1", "C2", "C3s", "C4", "C5", "sobel:2048", "enhance:2048")
# context only: the paper's own results on GTX745 / GTX680 / K20c (not targets)
CONTEXT = {"paper_geomean_speedup_max": 2.52, "paper_geomean_speedup_max_app": "Unsharp",
           "paper_harris_geomean_speedup": 1.208,
           "source": "PAPER.md:25-26, 1473-1481 (optimized vs baseline, three Nvidia GPUs)",
           "note": "fusion vs unfused on other hardware; compare with fused_vs_unfused here, not with value"}


def alg_bytes_per_px(spec: dict, blocks) -> int:
    """Algorithmic DRAM bytes per pixel of a plan: every launched
    block kernel reads each external image once and writes its sink once (4 B per
    pixel per image for f32 and for u8x4); halo re-reads excluded."""
    n_in, ops = spec["n_inputs"], spec["ops"]
    tot = 0
    for ks in blocks:
        inside = {n_in + k for k in ks}
        ext = {i for k in ks for i in ops[k]["inputs"] if i not in inside}
        tot += 4 * len(ext) + 4
    return tot


def workload_spec(cfg: str):
    """A BASELINE config name (C1..C5), or workload:size for a square extra app."""
    from kf_inputs import pipelines as P
    if ":" in cfg:
        wl, n = cfg.split(":")
        return P.WORKLOADS[wl](int(n), int(n)), 7
    return P.config(cfg)


def host_cpu() -> dict:
    """nproc and the lscpu model of this host (the CPU baseline's machine)."""
    model = None
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return {"nproc": os.cpu_count(), "model": model}


def load_peaks() -> dict:
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            d = json.load(f)
        return {"hbm_gbs": float(d["hbm_gbs"]), "source": "MEASURED_PEAKS.json hbm_gbs (measured copy)"}
    except Exception:
        return {"hbm_gbs": 6650.0, "source": "fallback 6.65 TB/s (B200_PROFILING.md)"}


def ncu_inst(cfg: str, plan: str):
    """warp instructions per pixel of the fused kernel from a committed ncu capture, if any."""
    path = os.path.join(ROOT, "profiles", "ncu_inst.json")
    try:
        with open(path) as f:
            return json.load(f).get(f"{cfg}:{plan}")
    except Exception:
        return None


def make_plan(p, kind):
    if kind == "unfused":
        return p.plan_unfused()
    if kind == "basic":
        return p.plan_basic("paper")
    return p.plan_fusion(kind)


def ncu_traffic(cfg: str, plan: str):
    """dram bytes per launch from the committed ncu --set full summary, if any."""
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(path) as f:
            d = json.load(f)
        return d.get(f"{cfg}:{plan}")
    except Exception:
        return None


class ClockSampler:
    """NVML samples of SM clock and throttle reasons during the timed region."""
    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
               0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
               0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, device: int):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _sample(self):
        nv = self.nv
        self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
        r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
        for bit, name in self.REASONS.items():
            if r & bit and name != "gpu_idle":
                self.reasons.add(name)

    def _loop(self):
        while not self._stop.is_set():
            try:
                self._sample()
            except Exception:
                return
            time.sleep(0.002)

    def __enter__(self):
        if self.nv:
            self.t = threading.Thread(target=self._loop, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.nv:
            self._stop.set()
            self.t.join()
            if not self.samples:
                self._sample()

    def summary(self) -> dict:
        if not self.nv:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvml unavailable"]}
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ----------------------------------------------------------------- reference


def cpu_oracle_run(spec: dict, seed: int, threads: int, rows: int | None = None) -> tuple[float, int, int]:
    """Times the unfused oracle on the workload (or its first `rows` rows as a
    smaller image of the same width); returns (seconds, pixels, threads used)."""
    from kf_inputs import gen
    from kf_inputs import pipelines as P
    from oracle import oracle as O
    if rows is not None and rows < spec["height"]:
        spec = P.WORKLOADS[spec["name"]](spec["width"], rows)
    used = O.set_threads(threads)
    ins = [gen.image(spec["dtype"], seed + 101 * j, spec["width"], spec["height"]) for j in range(spec["n_inputs"])]
    t = time.perf_counter()
    O.run(spec, ins)
    return time.perf_counter() - t, spec["width"] * spec["height"], used


REF_BUDGET_S = 150.0   # reference arm: longest run of whole-image steps before it samples row bands


def run_reference(args, cfg_name, spec, seed) -> None:
    """The reference arm: the unfused fp64 oracle on ALL host cores (OpenMP over
    rows), each step one whole image of the headline workload (same config)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    # Each step is the whole image unless --steps/--warmup would make the run
    # longer than REF_BUDGET_S; then every step is the same-width band of the
    # image's first `rows` rows, sized to the budget (a bounded sample).
    t_full, _, _ = cpu_oracle_run(spec, seed, 0)   # first warm-up step, whole image
    H = spec["height"]
    n_rest = max(1, args.warmup - 1 + args.steps)
    rows = H if n_rest * t_full <= REF_BUDGET_S else max(64, int(H * REF_BUDGET_S / (n_rest * t_full)) // 8 * 8)
    for _ in range(args.warmup - 1):
        cpu_oracle_run(spec, seed, 0, rows)
    tot, px, used = 0.0, 0, 1
    for _ in range(args.steps):
        dt, n, used = cpu_oracle_run(spec, seed, 0, rows)
        tot += dt
        px += n
    v = px / tot / 1e6
    whole = rows >= H
    sample = (f"the whole {spec['width']}x{spec['height']} {spec['name']} image per step (same config as the GPU arm)"
              if whole else f"the first {rows} rows ({spec['width']}x{rows}) of the {spec['width']}x{H} "
              f"{spec['name']} image per step: {args.steps} whole-image steps would exceed {REF_BUDGET_S:.0f} s")
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": round(v, 4), "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(tot / args.steps * 1e3, 3),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
        "data": DATA, "config": config_dict(cfg_name, spec, "unfused-oracle", {"l2": "n/a: host oracle"}),
        "cpu_baseline": {"value": round(v, 4), "unit": UNIT, "cores": used, "kind": "oracle", "sample": sample,
                         "host": host_cpu(), "parallel": "OpenMP over the rows of each kernel"},
        "e2e": {"value": round(v, 4), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "same_config": whole,
    }))


def config_dict(cfg_name, spec, plan, extra=None) -> dict:
    d = {"workload": f"{cfg_name}: {spec['name']} {spec['width']}x{spec['height']} {spec['dtype']}",
         "width": spec["width"], "height": spec["height"], "plan": plan,
         "l2": "4 rotating input/output buffer sets (512 MiB) > 126 MB L2"}
    if extra:
        d.update(extra)
    return d


# --------------------------------------------------------------------- GPU


def time_plan(plan, ins, outs, steps, warmup, stream, torch):
    """Times exactly `steps` kf_run calls (one step = one whole plan over one
    image, rotating over the buffer sets).  The steps are captured once into a
    CUDA graph so that the host-side launch cost of the ctypes binding is out of
    the timed region; the graph replay is bracketed by CUDA events on the
    launching stream.  Returns ms per step."""
    n = len(ins)
    with torch.cuda.stream(stream):
        for i in range(warmup):
            plan.run([ins[i % n]], [outs[i % n]], stream)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=stream):
        for i in range(steps):
            plan.run([ins[i % n]], [outs[i % n]], stream)
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(stream):                  # replay() launches on the current stream
        g.replay()                                   # warm replay (untimed)
        torch.cuda.synchronize()
        t0.record(stream)
        g.replay()
        t1.record(stream)
    torch.cuda.synchronize()
    return t0.elapsed_time(t1) / steps


FRAMES = 8   # frames per kf_run_batch call in the `frames` measurement


def time_batch(plan, ins, outs, frames, steps, stream, torch):
    """Times a stream of independent frames through kf_run_batch: `steps` frames
    as ceil(steps / frames) batch calls over `frames` disjoint buffer sets,
    captured into one CUDA graph like time_plan.  Returns ms per frame."""
    fi = [[x] for x in ins[:frames]]
    fo = [[x] for x in outs[:frames]]
    nb = max(1, -(-steps // frames))
    with torch.cuda.stream(stream):
        for _ in range(2):
            plan.run_batch(fi, fo, stream)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=stream):
        for _ in range(nb):
            plan.run_batch(fi, fo, stream)
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(stream):
        g.replay()
        torch.cuda.synchronize()
        t0.record(stream)
        g.replay()
        t1.record(stream)
    torch.cuda.synchronize()
    return t0.elapsed_time(t1) / (nb * frames)


def frames_block(plan, host, oshape, tdt, px, ab, single_ms, steps, stream, torch, what=True) -> dict:
    """A stream of independent frames of the workload through kf_run_batch
    (frames after the first overlap the previous frame's tail):
    ms per frame, Mpixel/s and HBM fraction, beside the single-image kf_run."""
    ins = [torch.from_numpy(host).cuda() for _ in range(FRAMES)]
    outs = [torch.empty(oshape, dtype=tdt, device="cuda") for _ in range(FRAMES)]
    ms = time_batch(plan, ins, outs, FRAMES, steps, stream, torch)
    del ins, outs
    torch.cuda.empty_cache()
    peak = load_peaks()["hbm_gbs"]
    d = {"frames_per_call": FRAMES, "ms_per_frame": round(ms, 5), "mpix_s": round(px / (ms * 1e-3) / 1e6, 1),
         "hbm_frac": round(ab * px / (ms * 1e-3) / 1e9 / peak, 4),
         "vs_single_kf_run": round(single_ms / ms, 3)}
    if what:
        d["what"] = ("kf_run_batch over independent frames (disjoint buffers): frame f+1's CTAs fill the SM "
                     "slots frame f's tail leaves idle (programmatic dependent launch); not the headline, "
                     "which is one kf_run per image")
    return d


def bench_single(args, cfg_name, spec, seed) -> None:
    import torch

    from kf_inputs import gen
    from paper_conf_cgo_qiaorht19_b200 import kfuse as K

    dev = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(dev)
    W, H = spec["width"], spec["height"]
    px = W * H
    host = gen.image(spec["dtype"], seed, W, H)
    tdt = torch.float32 if spec["dtype"] == "f32" else torch.uint8
    oshape = (H, W) if spec["dtype"] == "f32" else (H, W, 4)
    nsets = 4
    ins = [torch.from_numpy(host).cuda() for _ in range(nsets)]
    outs = [torch.empty(oshape, dtype=tdt, device="cuda") for _ in range(nsets)]
    stream = torch.cuda.Stream()
    results = {}
    plans = {}
    for kind in PLANS:
        p = K.Pipeline.from_spec(spec)
        plan = make_plan(p, kind)
        plan.prepare()
        plans[kind] = (p, plan)
    # headline plan last, with clocks sampled during its timed region
    order = [k for k in PLANS if k != args.plan] + [args.plan]
    clocks = None
    for kind in order:
        p, plan = plans[kind]
        if kind == args.plan:
            with ClockSampler(dev) as cs:
                ms = time_plan(plan, ins, outs, args.steps, args.warmup, stream, torch)
            clocks = cs.summary()
        else:
            ms = time_plan(plan, ins, outs, max(50, args.steps // 4), args.warmup, stream, torch)
        ab = alg_bytes_per_px(spec, plan.blocks)
        results[kind] = {"ms_per_step": round(ms, 5), "mpix_s": round(px / (ms * 1e-3) / 1e6, 1),
                         "launches": plan.num_launches, "alg_bytes_per_px": ab,
                         "alg_gbs": round(ab * px / (ms * 1e-3) / 1e9, 1)}
    head = results[args.plan]
    # distribution over repeated timed replays (the paper reports the median of
    # 500 runs): 11 replays of min(K, 100) steps each, ms/step
    if not args.no_extra:
        reps = sorted(time_plan(plans[args.plan][1], ins, outs, min(args.steps, 100), 1, stream, torch) for _ in range(11))
        head["replays"] = {"n": 11, "steps_each": min(args.steps, 100), "median_ms": round(reps[5], 5),
                           "min_ms": round(reps[0], 5), "iqr_ms": round(reps[8] - reps[2], 5)}
    peaks = load_peaks()
    _, hplan = plans[args.plan]
    ab = head["alg_bytes_per_px"] or 8
    # the headline plan is one launch per step, so the step time of the graph
    # replay is that kernel's average launch duration
    achieved = ab * px / (head["ms_per_step"] * 1e-3) / 1e9
    traffic = ncu_traffic(cfg_name, args.plan)
    roofline = {"bound": "hbm", "achieved": round(achieved, 1), "peak": peaks["hbm_gbs"], "unit": "GB/s",
                "frac": round(achieved / peaks["hbm_gbs"], 4), "traffic": traffic,
                "peak_source": peaks["source"],
                "per_launch": f"{ab} B/px x {px} px = {ab * px} algorithmic bytes per launch"}
    # Same-size memory floor: the framework's own 1-in/1-out copy kernel (same
    # launch path, streaming loop and buffer rotation) over the same pixel count.
    # Context for `frac`: at these sizes the ramp and drain of a ~20 us kernel
    # keep even a copy below the large-transfer copy peak.
    if not args.no_extra:
        roofline["copy_floor"] = copy_floor(W, H, ins, stream, torch, ab * px)
        roofline["copy_floor"]["fused_over_copy"] = round(roofline["copy_floor"]["ms_per_step"] / head["ms_per_step"], 4)
    frames = None
    if not args.no_extra and hplan.num_launches == 1:
        frames = frames_block(hplan, host, oshape, tdt, px, ab, head["ms_per_step"], args.steps, stream, torch)
    # end to end through the public API with host buffers (pinned)
    e2e_steps = max(3, min(args.steps, 20))
    hin = torch.from_numpy(host).pin_memory()
    hout = torch.empty(oshape, dtype=tdt).pin_memory()
    for _ in range(2):
        hplan.run_host([hin], [hout], stream)
    torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(e2e_steps):
        hplan.run_host([hin], [hout], stream)
    e2e_sync_s = (time.perf_counter() - t) / e2e_steps
    # a stream of images through kf_run_host_async (the next image's uploads
    # overlap this one's downloads); every step still uploads its input from
    # pinned host memory and downloads its result; synchronised at the end
    for _ in range(2):
        hplan.run_host_async([hin], [hout], stream)
    stream.synchronize()
    t = time.perf_counter()
    for _ in range(e2e_steps):
        hplan.run_host_async([hin], [hout], stream)
    stream.synchronize()
    e2e_s = (time.perf_counter() - t) / e2e_steps
    e2e = {"value": round(px / e2e_s / 1e6, 1), "unit": UNIT, "h2d_bytes_per_step": int(hin.numel() * hin.element_size()),
           "d2h_bytes_per_step": int(hout.numel() * hout.element_size()), "steps": e2e_steps,
           "api": "kf_run_host_async per image, one synchronisation after the last",
           "per_call_sync": {"value": round(px / e2e_sync_s / 1e6, 1), "unit": UNIT,
                             "api": "kf_run_host (synchronises every call)"}}
    if not args.no_extra:
        e2e["pcie_floor"] = pcie_floor(hin, hout, px, torch)
    # CPU baseline: the unfused oracle on this box's host, one full image, on all
    # cores (OpenMP over rows) and on one thread (SURVEY §8(d) "two modes")
    cpu = None
    if not args.no_cpu:
        rows = None if spec["dtype"] == "f32" else 256
        dt, n, used = cpu_oracle_run(spec, seed, 0, rows)
        dt1, n1, _ = cpu_oracle_run(spec, seed, 1, rows)
        img = f"{W}x{rows or H}"
        cpu = {"value": round(n / dt / 1e6, 3), "unit": UNIT, "cores": used, "kind": "oracle",
               "sample": f"one {img} image of the workload, unfused fp64 oracle, OpenMP over rows on {used} threads",
               "host": host_cpu(),
               "single_thread": {"value": round(n1 / dt1 / 1e6, 3), "unit": UNIT, "cores": 1,
                                 "sample": f"the same {img} image, 1 thread"}}
    del ins, outs
    extra = {} if args.no_extra else bench_extra(args, stream, torch, clocks)
    out = {
        "metric": METRIC, "value": head["mpix_s"], "unit": UNIT, "n_gpus": 1, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": head["ms_per_step"], "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f32" if spec["dtype"] == "f32" else "u8x4/int32", "data": DATA,
        "config": config_dict(cfg_name, spec, args.plan),
        "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
        "gpu_launches": args.steps * hplan.num_launches, "clocks": clocks,
        "plans": results,
        "fused_vs_unfused": round(results["unfused"]["ms_per_step"] / head["ms_per_step"], 3),
        "frames": frames,
        "context": CONTEXT,
        "workloads": extra,
    }
    print(json.dumps(out))


def pcie_floor(hin, hout, px, torch) -> dict:
    """The e2e leg's ceiling on this box: the same H2D and D2H byte counts as one
    step, copied concurrently on two streams with no kernel in between (what
    kf_run_host overlaps with its row bands).  Wall time over 5 repetitions."""
    d_in = torch.empty(hin.shape, dtype=hin.dtype, device="cuda")
    d_out = torch.empty(hout.shape, dtype=hout.dtype, device="cuda")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()

    def both():
        with torch.cuda.stream(s1):
            d_in.copy_(hin, non_blocking=True)
        with torch.cuda.stream(s2):
            hout.copy_(d_out, non_blocking=True)
        torch.cuda.synchronize()
    both()
    t = time.perf_counter()
    for _ in range(5):
        both()
    dt = (time.perf_counter() - t) / 5
    nb = hin.numel() * hin.element_size() + hout.numel() * hout.element_size()
    del d_in, d_out
    return {"value": round(px / dt / 1e6, 1), "unit": UNIT, "gbs_both_directions": round(nb / dt / 1e9, 1),
            "what": "H2D + D2H of one step's bytes, concurrent, no compute: the ceiling of e2e"}


def copy_floor(W, H, ins, stream, torch, fused_bytes) -> dict:
    """Times the `copy` diagnostic pipeline (one point kernel, out = in, 8 B/px)
    over W x H f32 pixels, exactly like the fused plan (graph replay, rotating
    buffer sets larger than L2).  A u8x4 image has the same 4 B/px."""
    from kf_inputs import pipelines as P
    from paper_conf_cgo_qiaorht19_b200 import kfuse as K
    n = len(ins)
    cin = [torch.empty((H, W), dtype=torch.float32, device="cuda").uniform_() for _ in range(n)]
    cout = [torch.empty_like(x) for x in cin]
    plan = K.Pipeline.from_spec(P.copy(W, H)).plan_fusion("b200")
    plan.prepare()
    ms = time_plan(plan, cin, cout, 200, 3, stream, torch)
    del cin, cout
    gbs = 8 * W * H / (ms * 1e-3) / 1e9
    return {"ms_per_step": round(ms, 5), "gbs": round(gbs, 1), "frac_of_peak": round(gbs / load_peaks()["hbm_gbs"], 4),
            "what": "the framework's own copy kernel (8 B/px) over the same pixel count"}


def bench_extra(args, stream, torch, clocks) -> dict:
    """The other BASELINE.json configs (C1 Harris 256^2, C2 Unsharp 2048^2, C3s
    ShiTomasi 4096^2, C4 deep10 7680x4320 u8x4), every plan, timed like the
    headline (CUDA-graph replay, rotating buffer sets larger than L2).  The fused
    plan gets its HBM fraction (algorithmic bytes) and, where a committed ncu
    capture gives its instruction count, its issue fraction (C4 is ALU-bound,
    SURVEY §8(d)): warp instructions / (148 SMs x 4 schedulers x SM clock)."""
    from kf_inputs import gen
    from kf_inputs import pipelines as P
    from paper_conf_cgo_qiaorht19_b200 import kfuse as K
    peaks = load_peaks()
    sm_hz = ((clocks or {}).get("sm_mhz") or 1965.0) * 1e6
    n_sm = torch.cuda.get_device_properties(torch.cuda.current_device()).multi_processor_count
    res = {}
    for cfg in EXTRA_CONFIGS:
        spec, seed = workload_spec(cfg)
        W, H = spec["width"], spec["height"]
        px = W * H
        host = gen.image(spec["dtype"], seed, W, H)
        tdt = torch.float32 if spec["dtype"] == "f32" else torch.uint8
        oshape = (H, W) if spec["dtype"] == "f32" else (H, W, 4)
        nsets = max(2, min(8, int(512e6 // (8 * px))))     # sets x (in + out) >= ~512 MB > L2 where possible
        ins = [torch.from_numpy(host).cuda() for _ in range(nsets)]
        outs = [torch.empty(oshape, dtype=tdt, device="cuda") for _ in range(nsets)]
        d = {"workload": f"{spec['name']} {W}x{H} {spec['dtype']}", "plans": {}}
        for kind in PLANS:
            p = K.Pipeline.from_spec(spec)
            plan = make_plan(p, kind)
            plan.prepare()
            steps = 6 if px > 1e8 else 20 if px > 2e7 else 100
            ms = time_plan(plan, ins, outs, steps, 3, stream, torch)
            ab = alg_bytes_per_px(spec, plan.blocks)
            d["plans"][kind] = {"ms_per_step": round(ms, 5), "mpix_s": round(px / (ms * 1e-3) / 1e6, 1),
                                "launches": plan.num_launches, "blocks": len(plan.blocks), "alg_bytes_per_px": ab,
                                "hbm_frac": round(ab * px / (ms * 1e-3) / 1e9 / peaks["hbm_gbs"], 4)}
        f = d["plans"]["b200"]
        d["fused_vs_unfused"] = round(d["plans"]["unfused"]["ms_per_step"] / f["ms_per_step"], 3)
        d["basic_vs_unfused"] = round(d["plans"]["unfused"]["ms_per_step"] / d["plans"]["basic"]["ms_per_step"], 3)
        d["paper_vs_unfused"] = round(d["plans"]["unfused"]["ms_per_step"] / d["plans"]["paper"]["ms_per_step"], 3)
        if px >= 1 << 22:
            d["copy_floor"] = copy_floor(W, H, ins, stream, torch, 8 * px)
            d["copy_floor"]["fused_over_copy"] = round(d["copy_floor"]["ms_per_step"] / f["ms_per_step"], 4)
        fplan = make_plan(K.Pipeline.from_spec(spec), "b200")
        if fplan.num_launches == 1 and FRAMES * 8 * px < 40e9:
            del ins, outs
            torch.cuda.empty_cache()
            steps = 16 if px > 1e8 else 40 if px > 2e7 else 200
            d["frames"] = frames_block(fplan, host, oshape, tdt, px, alg_bytes_per_px(spec, fplan.blocks),
                                       f["ms_per_step"], steps, stream, torch, what=False)
            ins, outs = [], []
        ipp = ncu_inst(cfg, "b200")
        if ipp:
            issue = ipp * px / (f["ms_per_step"] * 1e-3)
            d["issue"] = {"bound": "alu", "warp_inst_per_px": ipp, "achieved": round(issue / 1e9, 1),
                          "peak": round(n_sm * 4 * sm_hz / 1e9, 1), "unit": "G warp-inst/s",
                          "frac": round(issue / (n_sm * 4 * sm_hz), 4),
                          "source": "profiles/ncu_inst.json (ncu smsp__inst_executed.sum / px)"}
        res[cfg] = d
        del ins, outs
        torch.cuda.empty_cache()
    return res


def _band_run(args, gspec, seed, plan, rank, world, dev, torch, dist, KD, stream, side, e2e=False) -> dict:
    """Times `args.steps` row-band steps of one global image on this rank: the
    halo exchange with the neighbours behind the band's core rows, then the edge
    strips.  Returns the per-rank timing (max over ranks), the transport, the
    halo bytes and an exchange-free compute-only time (the same band computed
    from pre-filled halo rows) that tells whether the exchange was hidden."""
    from kf_inputs import gen
    W, Htot = gspec["width"], gspec["height"]
    band = KD.partition(Htot, world, rank, plan.halo_rows)
    host = gen.image(gspec["dtype"], seed, W, Htot, band.in0, band.in1)
    tdt = torch.float32 if gspec["dtype"] == "f32" else torch.uint8
    nsets = 4
    ins = [torch.from_numpy(host).cuda() for _ in range(nsets)]
    oshape = (band.rows, W) if gspec["dtype"] == "f32" else (band.rows, W, 4)
    outs = [torch.empty(oshape, dtype=tdt, device="cuda") for _ in range(nsets)]
    # halo transport: peer memory (CUDA IPC mappings over NVLink, device-counter
    # sync, whole steps captured in a CUDA graph) or NCCL send/recv (eager)
    mode = os.environ.get("KFUSE_HALO", "peer")
    halo, note = None, ""
    if mode == "peer":
        try:
            halo = KD.PeerHalo(band, ins)
        except Exception as e:   # e.g. no IPC between the ranks: fall back to NCCL
            mode, note = "nccl", f"peer setup failed ({type(e).__name__}: {e}); "
        # every rank must use the same transport: peer only if it worked everywhere
        agree = torch.tensor([1 if mode == "peer" else 0], dtype=torch.int32,
                             device="cuda" if dist.get_backend() == "nccl" else "cpu")
        dist.all_reduce(agree, op=dist.ReduceOp.MIN)
        if int(agree.item()) == 0 and mode == "peer":
            mode, halo, note = "nccl", None, "peer setup failed on another rank; "
    ref_out = torch.empty_like(outs[0])
    plan.run_band(band.row0, band.row1, [ins[0]], band.in0, band.in1, [ref_out], stream)
    torch.cuda.synchronize()
    if mode == "peer" and (halo.up is not None or halo.down is not None):
        # Self-check on this hardware before timing: the buffers were generated
        # with their halo rows, so kf_run_band over them is the reference.  Poison
        # the halo rows, run one peer step, and require the same bits; else every
        # rank falls back to NCCL (and says so in the JSON line).
        ok = 1
        try:
            t_, n_ = band.top, band.rows
            if gspec["dtype"] == "f32":
                ins[0][:t_].fill_(float("nan"))
                ins[0][t_ + n_:].fill_(float("nan"))
            else:
                ins[0][:t_].fill_(77)
                ins[0][t_ + n_:].fill_(77)
            chk = torch.empty_like(outs[0])
            dist.barrier()
            halo.step(plan, 0, [chk], stream, side)
            torch.cuda.synchronize()
            ok = int(halo.errors() == 0 and torch.equal(chk, ref_out))
        except Exception as e:   # noqa: BLE001 -- any failure means: do not use the peer path
            note += f"peer self-check raised {type(e).__name__}; "
            ok = 0
        agree = torch.tensor([ok], dtype=torch.int32, device="cuda" if dist.get_backend() == "nccl" else "cpu")
        dist.all_reduce(agree, op=dist.ReduceOp.MIN)
        if int(agree.item()) == 0:
            mode, halo, note = "nccl", None, note + "peer self-check failed; "
            ins[0].copy_(torch.from_numpy(host).to(ins[0].device))   # restore the halo rows
    (c0, c1), edges = KD.split_rows(band)
    exch = world > 1 and plan.halo_rows > 0 and (halo is None or halo.up is not None or halo.down is not None)
    launches_per_step = plan.num_launches * ((1 if c1 > c0 else 0) + len(edges)) + \
        (2 if exch and mode == "peer" else 0)

    def step(i):
        if mode == "peer":   # core rows || (signal, halo pull over peer loads), then the edge strips
            halo.step(plan, i % nsets, [outs[i % nsets]], stream, side)
        else:                # NCCL send/recv overlapped with the core rows
            KD.run_step_overlapped(plan, band, [ins[i % nsets]], [outs[i % nsets]], side)

    def timed(fn, graphable):
        for i in range(args.warmup):
            fn(i)
        torch.cuda.synchronize()
        graph = None
        if graphable:   # every rank captures the same steps; the counters synchronise the replays
            graph = torch.cuda.CUDAGraph()
            with torch.cuda.graph(graph, stream=stream):
                for i in range(args.steps):
                    fn(i)
            torch.cuda.synchronize()
            dist.barrier()
            with torch.cuda.stream(stream):   # one untimed replay: the first launch uploads the graph
                graph.replay()
            torch.cuda.synchronize()
        dist.barrier()
        t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with ClockSampler(dev) as cs:
            t0.record(stream)
            if graph is not None:
                graph.replay()
            else:
                for i in range(args.steps):
                    fn(i)
            t1.record(stream)
            torch.cuda.synchronize()
        dist.barrier()
        ms = torch.tensor([t0.elapsed_time(t1) / args.steps], device="cuda")
        dist.all_reduce(ms, op=dist.ReduceOp.MAX)
        del graph
        return float(ms.item()), cs.summary()

    ms, clocks = timed(step, mode == "peer")
    if halo is not None:
        bad = torch.tensor([halo.errors()], device="cuda")
        dist.all_reduce(bad, op=dist.ReduceOp.MAX)
        if int(bad.item()):
            raise RuntimeError("peer halo: a counter wait timed out")
    # the same band work without any exchange (halo rows already in place): if
    # the step costs no more than this, the exchange was hidden behind the core
    for k in range(nsets):
        ins[k].copy_(torch.from_numpy(host).to(ins[k].device))

    def compute_only(i):
        plan.run_band(band.row0, band.row1, [ins[i % nsets]], band.in0, band.in1, [outs[i % nsets]], stream)
    ms_c, _ = timed(compute_only, True)
    rb = W * 4
    halo_bytes = (band.top + band.bottom) * rb * gspec["n_inputs"] if exch else 0
    hb = torch.tensor([halo_bytes], dtype=torch.float64, device="cuda")
    dist.all_reduce(hb, op=dist.ReduceOp.SUM)
    res = {"ms": ms, "clocks": clocks, "mode": mode, "note": note, "band": band, "plan": plan,
           "launches_per_step": launches_per_step,
           "exchange": {"transport": ("peer-memory halo pull (CUDA IPC / NVLink P2P, device-counter sync), steps "
                                      "replayed from a CUDA graph") if mode == "peer" else
                        "NCCL send/recv overlapped with the core rows",
                        "halo_rows": plan.halo_rows, "halo_bytes_per_step_this_rank": halo_bytes,
                        "halo_bytes_per_step_all_ranks": int(hb.item()),
                        "step_ms": round(ms, 5), "compute_only_ms": round(ms_c, 5),
                        "exchange_overhead_frac": round(ms / ms_c - 1.0, 4),
                        "hidden": bool(ms <= ms_c * 1.03)}}
    if e2e:
        # end to end through the public API: each step uploads the band's own rows
        # from pinned host memory, runs the step (halo exchange + fused kernels)
        # and downloads the band's output; max over ranks of the wall time
        hin = torch.from_numpy(host).pin_memory()
        hout = torch.empty(oshape, dtype=tdt).pin_memory()
        t, n = band.top, band.rows
        e2e_steps = max(3, min(args.steps, 20))

        def e2e_step():
            if halo is not None:
                halo.wait_consumed(stream)        # the neighbours pulled the previous rows
            ins[0][t:t + n].copy_(hin[t:t + n], non_blocking=True)
            if halo is not None:
                halo.step(plan, 0, [outs[0]], stream, side)
            else:
                KD.run_step_overlapped(plan, band, [ins[0]], [outs[0]], side)
            hout.copy_(outs[0], non_blocking=True)
            stream.synchronize()

        e2e_step()
        dist.barrier()
        tw = time.perf_counter()
        for _ in range(e2e_steps):
            e2e_step()
        e2e_s = torch.tensor([(time.perf_counter() - tw) / e2e_steps], device="cuda")
        dist.all_reduce(e2e_s, op=dist.ReduceOp.MAX)
        res["e2e"] = {"value": round(W * Htot / float(e2e_s.item()) / 1e6, 1), "unit": UNIT,
                      "h2d_bytes_per_step": int(n * hin[0].numel() * hin.element_size()),
                      "d2h_bytes_per_step": int(hout.numel() * hout.element_size()), "steps": e2e_steps,
                      "note": "per rank, max over ranks"}
    if halo is not None:   # drop the peer mappings on every rank before any rank frees its buffers
        halo.close()
        dist.barrier()
    res["_keep"] = (halo, ins, outs)   # freed by the caller after every rank is done
    return res


def bench_multi(args, cfg_name, spec, seed) -> None:
    import torch
    import torch.distributed as dist

    from kf_inputs import pipelines as P
    from paper_conf_cgo_qiaorht19_b200 import dist as KD
    from paper_conf_cgo_qiaorht19_b200 import kfuse as K

    # KFUSE_DIST_BACKEND=gloo and KFUSE_BENCH_DEVICE=0 let a 2-rank smoke run share one GPU (tests only)
    dist.init_process_group(os.environ.get("KFUSE_DIST_BACKEND", "nccl"))
    rank, world = dist.get_rank(), dist.get_world_size()
    dev = int(os.environ.get("KFUSE_BENCH_DEVICE", os.environ.get("LOCAL_RANK", rank)))
    torch.cuda.set_device(dev)
    # NCCL prints its version banner on stdout when the first communicator is
    # created: create it now with stdout pointed at stderr (stdout carries the
    # one JSON line)
    sys.stdout.flush()
    saved = os.dup(1)
    os.dup2(2, 1)
    try:
        dist.barrier()
    finally:
        sys.stdout.flush()
        os.dup2(saved, 1)
        os.close(saved)
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    side = torch.cuda.Stream()
    peaks = load_peaks()
    dtype = "f32" if spec["dtype"] == "f32" else "u8x4/int32"

    # headline: weak scaling, one band of the config's size per GPU
    W, Hb = spec["width"], spec["height"]
    gspec = P.WORKLOADS[spec["name"]](W, Hb * world)
    plan = make_plan(K.Pipeline.from_spec(gspec), args.plan)
    plan.prepare()
    weak = _band_run(args, gspec, seed, plan, rank, world, dev, torch, dist, KD, stream, side, e2e=True)
    # BASELINE C5: one 16384^2 Harris image split into `world` bands (strong scaling)
    strong = None
    if not args.no_extra and cfg_name != "C5":
        c5, c5seed = P.config("C5")
        c5plan = make_plan(K.Pipeline.from_spec(c5), args.plan)
        c5plan.prepare()
        strong = _band_run(args, c5, c5seed, c5plan, rank, world, dev, torch, dist, KD, stream, side)

    def summary(r, g):
        px_all = g["width"] * g["height"]
        band = r["band"]
        ab = alg_bytes_per_px(g, r["plan"].blocks)
        ach = ab * (band.rows * g["width"]) / (r["ms"] * 1e-3) / 1e9
        return px_all, {"bound": "hbm", "achieved": round(ach, 1), "peak": peaks["hbm_gbs"], "unit": "GB/s",
                        "frac": round(ach / peaks["hbm_gbs"], 4), "traffic": None,
                        "peak_source": peaks["source"], "note": "per GPU (largest band), step time incl. halo exchange"}

    if rank == 0:
        px, roof = summary(weak, gspec)
        out = {
            "metric": METRIC, "value": round(px / (weak["ms"] * 1e-3) / 1e6, 1), "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(weak["ms"], 5),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": dtype, "data": DATA,
            "config": config_dict(cfg_name, gspec, args.plan,
                                  {"parallelism": f"row bands x{world}, halo {plan.halo_rows} rows: "
                                                  f"{weak['note']}{weak['exchange']['transport']}",
                                   "band": f"{Hb}x{W} per GPU"}),
            "roofline": roof, "cpu_baseline": None, "e2e": weak["e2e"],
            "gpu_launches": args.steps * weak["launches_per_step"], "clocks": weak["clocks"],
            "exchange": weak["exchange"], "context": CONTEXT,
        }
        if strong is not None:
            c5, _ = P.config("C5")
            px5, roof5 = summary(strong, c5)
            out["strong_c5"] = {
                "workload": f"C5: harris {c5['width']}x{c5['height']} f32, {world} row bands", "scaling": "strong",
                "value": round(px5 / (strong["ms"] * 1e-3) / 1e6, 1), "unit": UNIT,
                "ms_per_step": round(strong["ms"], 5), "rows_per_gpu": strong["band"].rows,
                "roofline": roof5, "exchange": strong["exchange"],
                "gpu_launches": args.steps * strong["launches_per_step"]}
        print(json.dumps(out))
    dist.barrier()
    del weak, strong
    torch.cuda.synchronize()
    dist.destroy_process_group()
    # Leave without the interpreter's teardown: torch's CUDA-IPC bookkeeping of
    # the exchanged buffers can crash at exit after everything above has been
    # released and the result printed (seen as SIGSEGV at world 1).
    sys.stdout.flush()
    sys.stderr.flush()
    os._exit(0)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=1000)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="kfuse", choices=["kfuse", "reference"])
    ap.add_argument("--config", default="C3")
    ap.add_argument("--plan", default="b200", choices=list(PLANS))
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--no-extra", action="store_true", help="skip the other BASELINE configs")
    ap.add_argument("--force-multi", action="store_true", help="run the row-band (torchrun) path even at world 1")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    from kf_inputs import pipelines as P
    spec, seed = P.config(args.config)
    if args.impl == "reference":
        run_reference(args, args.config, spec, seed)
        return
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world > 1 or args.force_multi:
        bench_multi(args, args.config, spec, seed)
    else:
        bench_single(args, args.config, spec, seed)


if __name__ == "__main__":
    main()

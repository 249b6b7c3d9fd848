"""GPU parity: the fused sm_100a kernels (through the C-ABI) against the unfused
CPU oracle on the same seeded inputs.

Bar: u8x4 pipelines bit-exact; f32 pipelines
max|gpu - oracle| / max|oracle| <= 1e-5 (the oracle is fp64, the GPU f32).
"""
import random

import numpy as np
import pytest
import torch

from kf_inputs import gen
from kf_inputs import pipelines as P
from oracle import oracle as O
from oracle import planner as PL
from paper_conf_cgo_qiaorht19_b200 import kfuse as K

pytestmark = pytest.mark.gpu
TOL = 1e-5


def _inputs(spec, seed):
    return [gen.image(spec["dtype"], seed + 101 * j, spec["width"], spec["height"]) for j in range(spec["n_inputs"])]


def _alloc(spec):
    H, W = spec["height"], spec["width"]
    dt = torch.float32 if spec["dtype"] == "f32" else torch.uint8
    shape = (H, W) if spec["dtype"] == "f32" else (H, W, 4)
    return [torch.empty(shape, dtype=dt, device="cuda") for _ in spec["outputs"]]


def make_plan(spec, kind):
    p = K.Pipeline.from_spec(spec)
    if kind == "unfused":
        return p.plan_unfused()
    if kind == "whole":
        return p.plan_from_blocks([0] * len(spec["ops"]))
    return p.plan_fusion(kind)


def run_gpu(spec, plan, ins):
    d_in = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in ins]
    outs = _alloc(spec)
    plan.run(d_in, outs)
    torch.cuda.synchronize()
    return [o.cpu().numpy() for o in outs]


def check(spec, got, ref, what=""):
    if spec["dtype"] == "u8x4":
        bad = np.argwhere(np.any(got != ref, axis=-1))
        assert len(bad) == 0, f"{what}: {len(bad)} pixels differ, first {bad[:5].tolist()}"
        return 0.0
    got = got.astype(np.float64)
    scale = np.abs(ref).max()
    err = np.abs(got - ref).max() / (scale if scale > 0 else 1.0)
    assert np.all(np.isfinite(got)) == np.all(np.isfinite(ref))
    assert err <= TOL, f"{what}: normalised error {err:.3g} > {TOL}"
    return err


def parity(spec, kind, seed=1):
    ins = _inputs(spec, seed)
    plan = make_plan(spec, kind)
    got = run_gpu(spec, plan, ins)
    ref = O.run(spec, ins)
    for g, o in zip(got, spec["outputs"]):
        check(spec, g, ref[o], f"{spec['name']} {kind} {spec['width']}x{spec['height']}")
    return plan


# --------------------------------------------------------------- workloads

@pytest.mark.parametrize("wl", ["harris", "shitomasi", "unsharp", "sobel", "enhance", "deep10"])
@pytest.mark.parametrize("kind", ["unfused", "paper", "b200"])
@pytest.mark.parametrize("size", [(67, 41), (256, 256)])
def test_workloads(wl, kind, size):
    parity(P.WORKLOADS[wl](*size), kind)


@pytest.mark.parametrize("mode", P.MODES)
@pytest.mark.parametrize("wl", ["harris", "deep10"])
def test_workloads_all_border_modes_fused(wl, mode):
    """Index exchange under every border mode (pad-once differs under
    clamp/constant for Harris and under every non-wrap mode for deep10)."""
    spec = P.WORKLOADS[wl](45, 37, mode=mode)
    plan = parity(spec, "b200")
    if mode != "repeat" or wl == "deep10":
        assert plan.num_launches == 1


def test_fig4_fused_on_gpu():
    """Fig. 4c through the fused GPU kernel: 763 at (0,0), 992 at (2,2)."""
    spec = P.fig4("clamp")
    img = np.array(P.FIG4_IMAGE, np.float32)
    plan = make_plan(spec, "whole")
    assert plan.num_launches == 1
    out = run_gpu(spec, plan, [img])[0]
    assert out[0, 0] == 763 and out[2, 2] == 992
    ref = O.run(spec, [img])[2]
    np.testing.assert_array_equal(out, ref)


@pytest.mark.parametrize("size", [(1, 1), (2, 3), (3, 2), (5, 5), (31, 9), (33, 17), (7, 70)])
@pytest.mark.parametrize("wl", ["harris", "deep10", "unsharp"])
def test_tiny_and_ragged_images(wl, size):
    """Images smaller than the halo (mirror folds repeatedly), ragged tiles."""
    for mode in ("clamp", "mirror", "mirror101", "constant", "repeat"):
        parity(P.WORKLOADS[wl](*size, mode=mode), "b200")


@pytest.mark.parametrize("seed", range(60))
def test_random_dags(seed):
    rng = random.Random(70000 + seed)
    dtype = rng.choice(["f32", "u8x4"])
    W, H = rng.choice([(1, 1), (4, 3), (9, 9), (33, 17), (70, 45), (129, 20)])
    spec = P.random_pipeline(rng, W, H, dtype, rng.randint(2, 8))
    for kind in ("unfused", "paper", "b200"):
        parity(spec, kind, seed)
    # the exhaustive optimum's partition as well (any legal partition must be exact)
    best, blocks = PL.brute_force(spec, PL.B200_PROFILE) if len(spec["ops"]) <= 7 else (None, None)
    if blocks:
        lab = [0] * len(spec["ops"])
        for b, ks in enumerate(blocks):
            for k in ks:
                lab[k] = b
        ins = _inputs(spec, seed)
        plan = K.Pipeline.from_spec(spec).plan_from_blocks(lab)
        got = run_gpu(spec, plan, ins)
        ref = O.run(spec, ins)
        for g, o in zip(got, spec["outputs"]):
            check(spec, g, ref[o], "brute-force partition")


# ------------------------------------------------------ full BASELINE sizes

def _sample_points(W, H, rng, n=1500):
    ys = list(rng.integers(0, H, n)) + [0, 0, H - 1, H - 1] + [0] * 20 + [H - 1] * 20 + list(range(min(H, 8)))
    xs = list(rng.integers(0, W, n)) + [0, W - 1, 0, W - 1] + list(rng.integers(0, W, 40)) + [0] * min(H, 8)
    return np.array(ys), np.array(xs)


@pytest.mark.parametrize("cfg", ["C2", "C3", "C3s", "C4"])
def test_full_size_sampled(cfg):
    """At BASELINE.json's full sizes, in the launch configuration bench.py times
    (B200-profile plan): sampled outputs against the recursive oracle, and the
    fused result against the unfused GPU run element by element."""
    spec, seed = P.config(cfg)
    ins = _inputs(spec, seed)
    fused = make_plan(spec, "b200")
    got = run_gpu(spec, fused, ins)[0]
    rng = np.random.default_rng(3)
    ys, xs = _sample_points(spec["width"], spec["height"], rng)
    ref = O.eval_points(spec, ins, spec["outputs"][0], ys, xs)
    if spec["dtype"] == "u8x4":
        np.testing.assert_array_equal(got[ys, xs], ref)
    else:
        scale = np.abs(ref).max()
        assert np.abs(got[ys, xs].astype(np.float64) - ref).max() / scale <= TOL
    unf = run_gpu(spec, make_plan(spec, "unfused"), ins)[0]
    if spec["dtype"] == "u8x4":
        np.testing.assert_array_equal(got, unf)
    else:
        d = np.abs(got.astype(np.float64) - unf.astype(np.float64)).max() / np.abs(unf).max()
        assert d <= TOL


# ---------------------------------------------------------- other entry points

@pytest.mark.parametrize("wl", ["harris", "deep10", "unsharp"])
@pytest.mark.parametrize("kind", ["unfused", "paper", "b200"])
@pytest.mark.parametrize("size", [(300, 200), (64, 1030), (40, 9)])
def test_run_host_equals_run(wl, kind, size):
    """kf_run_host (row-band pipelined H2D / compute / D2H) == kf_run, bit for bit."""
    spec = P.WORKLOADS[wl](*size)
    ins = _inputs(spec, 4)
    plan = make_plan(spec, kind)
    dev = run_gpu(spec, plan, ins)[0]
    out = np.empty_like(dev)
    plan.run_host([np.ascontiguousarray(a) for a in ins], [out])
    np.testing.assert_array_equal(out, dev)


def test_run_host_repeat_and_pinned():
    """REPEAT plans (one band) and pinned host buffers on a non-default stream."""
    spec = P.harris(256, 300, "repeat")
    ins = _inputs(spec, 5)
    plan = make_plan(spec, "b200")
    dev = run_gpu(spec, plan, ins)[0]
    hin = torch.from_numpy(np.ascontiguousarray(ins[0])).pin_memory()
    hout = torch.empty(dev.shape, dtype=torch.float32).pin_memory()
    s = torch.cuda.Stream()
    plan.run_host([hin], [hout], s)
    np.testing.assert_array_equal(hout.numpy(), dev)
    spec = P.harris(256, 1024)
    ins = _inputs(spec, 6)
    plan = make_plan(spec, "b200")
    dev = run_gpu(spec, plan, ins)[0]
    hin = torch.from_numpy(np.ascontiguousarray(ins[0])).pin_memory()
    hout = torch.empty(dev.shape, dtype=torch.float32).pin_memory()
    for _ in range(3):   # repeated calls reuse the staging buffers, streams and events
        plan.run_host([hin], [hout], s)
    np.testing.assert_array_equal(hout.numpy(), dev)


@pytest.mark.parametrize("wl", ["harris", "deep10", "unsharp"])
@pytest.mark.parametrize("kind", ["unfused", "paper", "b200"])
def test_bands_bit_identical(wl, kind):
    """Row bands (the multi-GPU decomposition, §8(e)) reproduce the full run bit for bit."""
    spec = P.WORKLOADS[wl](130, 97)
    ins = _inputs(spec, 8)
    plan = make_plan(spec, kind)
    full = run_gpu(spec, plan, ins)[0]
    H, R = spec["height"], plan.halo_rows
    cuts = [0, 13, 40, 41, 97]
    for r0, r1 in zip(cuts[:-1], cuts[1:]):
        a0, a1 = max(0, r0 - R), min(H, r1 + R)
        d_in = [torch.from_numpy(np.ascontiguousarray(x[a0:a1])).cuda() for x in ins]
        out = torch.empty((r1 - r0,) + full.shape[1:], dtype=torch.float32 if spec["dtype"] == "f32" else torch.uint8,
                          device="cuda")
        plan.run_band(r0, r1, d_in, a0, a1, [out])
        torch.cuda.synchronize()
        np.testing.assert_array_equal(out.cpu().numpy(), full[r0:r1])


@pytest.mark.parametrize("wl", ["harris", "deep10"])
@pytest.mark.parametrize("rank,world", [(0, 3), (1, 3), (2, 3), (0, 1)])
def test_overlapped_step_equals_full_run(wl, rank, world, monkeypatch):
    """dist.run_step_overlapped (core rows on a side stream while the halo is in
    flight, then the edge strips) reproduces the full run; the halo rows are
    pre-filled here, so the NCCL post is stubbed out."""
    from paper_conf_cgo_qiaorht19_b200 import dist as KD
    spec = P.WORKLOADS[wl](200, 150)
    ins = _inputs(spec, 12)
    plan = make_plan(spec, "b200")
    full = run_gpu(spec, plan, ins)[0]
    band = KD.partition(spec["height"], world, rank, plan.halo_rows)
    monkeypatch.setattr(KD, "_post_halos", lambda inputs, band, group=None: [])
    d_in = [torch.from_numpy(np.ascontiguousarray(a[band.in0:band.in1])).cuda() for a in ins]
    out = torch.empty((band.rows,) + full.shape[1:], dtype=d_in[0].dtype, device="cuda")
    KD.run_step_overlapped(plan, band, d_in, [out], torch.cuda.Stream())
    torch.cuda.synchronize()
    np.testing.assert_array_equal(out.cpu().numpy(), full[band.row0:band.row1])


def test_launch_count_matches_blocks():
    spec = P.harris(512, 512)
    for kind, n in (("unfused", 9), ("paper", 6), ("b200", 1)):
        assert make_plan(spec, kind).num_launches == n


# ------------------------------------------------ u8x4 SWAR form


@pytest.mark.parametrize("kind", ["unfused", "paper", "b200"])
@pytest.mark.parametrize("size", [(67, 41), (256, 96)])
def test_swar_matches_int32_and_oracle(kind, size, monkeypatch):
    """The SWAR form and the per-channel int32 form give the same bytes, and both
    equal the oracle (u8x4 parity is bit-exact)."""
    spec = P.swar_stress(*size)
    ins = _inputs(spec, 21)
    ref = O.run(spec, ins)[spec["outputs"][0]]
    outs = {}
    for sw in ("1", "0"):
        monkeypatch.setenv("KFUSE_SWAR", sw)
        plan = make_plan(spec, kind)
        outs[sw] = run_gpu(spec, plan, ins)[0]
        check(spec, outs[sw], ref, f"swar={sw} {kind} {size}")
    np.testing.assert_array_equal(outs["1"], outs["0"])


def test_c5_full_size_and_four_bands():
    """C5 (Harris 16384^2 f32, the multi-GPU config) at full size on one GPU:
    sampled outputs against the recursive oracle, and the 4-band decomposition
    (the 4-GPU row bands of §8(e), each band from its own input rows + halo)
    bit-identical to the whole-image run."""
    from paper_conf_cgo_qiaorht19_b200 import dist as KD
    spec, seed = P.config("C5")
    W, H = spec["width"], spec["height"]
    img = _inputs(spec, seed)[0]
    plan = make_plan(spec, "b200")
    d_in = torch.from_numpy(img).cuda()
    full = torch.empty((H, W), dtype=torch.float32, device="cuda")
    plan.run([d_in], [full])
    torch.cuda.synchronize()
    rng = np.random.default_rng(5)
    ys, xs = _sample_points(W, H, rng, n=800)
    ref = O.eval_points(spec, [img], spec["outputs"][0], ys, xs)
    got = full[torch.from_numpy(ys).cuda(), torch.from_numpy(xs).cuda()].cpu().numpy().astype(np.float64)
    assert np.abs(got - ref).max() / np.abs(ref).max() <= TOL
    for r in range(4):
        band = KD.partition(H, 4, r, plan.halo_rows)
        b_in = d_in[band.in0:band.in1].clone()
        b_out = torch.empty((band.rows, W), dtype=torch.float32, device="cuda")
        KD.run_band(plan, band, [b_in], [b_out])
        torch.cuda.synchronize()
        assert torch.equal(b_out, full[band.row0:band.row1]), f"band {r} differs"
        del b_in, b_out


# ------------------------------------------- halo rows over peer memory (§8(e))


def _peer_worker(rank, world, port, wl, graph, q):
    import os as _os
    import torch.distributed as dist
    from paper_conf_cgo_qiaorht19_b200 import dist as KD
    _os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)   # one GPU: the ranks share it, the IPC path is the same as across GPUs
        spec = P.WORKLOADS[wl](96, 130)
        W, H = spec["width"], spec["height"]
        plan = make_plan(spec, "b200")
        band = KD.partition(H, world, rank, plan.halo_rows)
        imgs = [gen.image(spec["dtype"], 40 + k, W, H) for k in range(3)]
        fulls = [run_gpu(spec, plan, [im])[0] for im in imgs]

        def own(k):   # a buffer with this band's own rows of image k, halo rows poisoned
            t = torch.from_numpy(np.ascontiguousarray(imgs[k][band.in0:band.in1])).cuda()
            t[:band.top] = 77
            t[band.top + band.rows:] = 77
            return t

        bufs = [own(0), own(1)]
        halo = KD.PeerHalo(band, bufs, spin_limit=1 << 24)
        side = torch.cuda.Stream() if graph else None
        outs = [torch.empty((band.rows,) + fulls[0].shape[1:], dtype=bufs[0].dtype, device="cuda") for _ in bufs]
        s = torch.cuda.Stream()
        ok = True
        if graph:
            for k in (0, 1):
                halo.step(plan, k, [outs[k]], s, side)   # warm-up (also outside the graph)
            s.synchronize()
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=s):
                for k in (0, 1):
                    halo.step(plan, k, [outs[k]], s, side)
            for _ in range(3):
                with torch.cuda.stream(s):
                    g.replay()
        else:
            for it in range(4):
                halo.step(plan, it % 2, [outs[it % 2]], s)
        s.synchronize()
        for k in (0, 1):
            ok &= bool(np.array_equal(outs[k].cpu().numpy(), fulls[k][band.row0:band.row1]))
        # overwrite set 0 with image 2 once both neighbours consumed it, then run again
        halo.wait_consumed(s)
        with torch.cuda.stream(s):
            bufs[0][band.top:band.top + band.rows].copy_(own(2)[band.top:band.top + band.rows])
        halo.step(plan, 0, [outs[0]], s)
        s.synchronize()
        ok &= bool(np.array_equal(outs[0].cpu().numpy(), fulls[2][band.row0:band.row1]))
        q.put((rank, ok, halo.errors()))
        halo.close()          # every rank drops its peer mappings before anyone frees
        dist.barrier()
        del halo, bufs, outs
        torch.cuda.synchronize()
        dist.barrier()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("wl,world,graph", [("harris", 2, False), ("harris", 3, True), ("deep10", 2, True)])
def test_peer_halo_steps(wl, world, graph):
    """dist.PeerHalo: halo rows pulled from the neighbours' buffers through CUDA
    IPC mappings, synchronised by device counters (kf_peer_signal / _pull / _wait),
    eager and captured in a CUDA graph, with rotating buffer sets and an
    overwrite guarded by wait_consumed -- bit-identical to the full-image run.
    The ranks share one GPU here; across GPUs the same mappings are NVLink peers."""
    import socket
    import torch.multiprocessing as mp
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_peer_worker, args=(r, world, port, wl, graph, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in procs:
        r, ok, err = q.get(timeout=300)
        res[r] = (ok, err)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert all(ok and err == 0 for ok, err in res.values()), res


@pytest.mark.parametrize("wl", ["harris", "shitomasi", "unsharp", "deep10"])
def test_strip_geometry_bit_identical(wl, monkeypatch):
    """The fused result does not depend on how the interior is cut into strips
    (peeled warm-up iterations vs the steady-state loop round identically)."""
    spec = P.WORKLOADS[wl](256, 240)
    ins = _inputs(spec, 9)
    plan = make_plan(spec, "b200")
    base = run_gpu(spec, plan, ins)[0]
    for ns in (2, 5, 40, 118):
        monkeypatch.setenv("KFUSE_NSTRIPS", str(ns))
        np.testing.assert_array_equal(run_gpu(spec, plan, ins)[0], base)


# Code-generation / launch knobs that change how the same arithmetic is
# scheduled: results must stay bit-identical to the default.
SAME_BITS = ["KFUSE_V8=1", "KFUSE_PERSIST=1", "KFUSE_QPTR=0", "KFUSE_LDS_PF=0", "KFUSE_CONST_W=0",
             "KFUSE_HEAVY_FIRST=0", "KFUSE_PRO_RP=0", "KFUSE_SMEM_ROWS=6"]


@pytest.mark.parametrize("wl", ["harris", "deep10", "unsharp"])
@pytest.mark.parametrize("knob", SAME_BITS)
def test_schedule_knobs_bit_identical(wl, knob, monkeypatch):
    spec = P.WORKLOADS[wl](200, 150)
    ins = _inputs(spec, 12)
    base = run_gpu(spec, make_plan(spec, "b200"), ins)[0]
    k, v = knob.split("=")
    monkeypatch.setenv(k, v)
    got = run_gpu(spec, make_plan(spec, "b200"), ins)[0]
    np.testing.assert_array_equal(got, base)


@pytest.mark.parametrize("wl", ["deep10", "harris"])
def test_rolled_edges_left_to_frame_still_exact(wl, monkeypatch):
    """KFUSE_ROLLED_EDGE_V=0 and a tiny code budget (rolled body) move rows between
    the streaming path and the frame tiles: u8x4 stays bit-exact, f32 within TOL."""
    spec = P.WORKLOADS[wl](130, 97)
    ins = _inputs(spec, 13)
    ref = O.run(spec, ins)[spec["outputs"][0]]
    for env in ({"KFUSE_ROLLED_EDGE_V": "0"}, {"KFUSE_CODE_BUDGET": "1000"},
                {"KFUSE_CODE_BUDGET": "1000", "KFUSE_ROLLED_EDGE_V": "0"}):
        for k, v in env.items():
            monkeypatch.setenv(k, v)
        got = run_gpu(spec, make_plan(spec, "b200"), ins)[0]
        check(spec, got, ref, f"{wl} {env}")
        for k in env:
            monkeypatch.delenv(k)

"""Bounds-checked runs of the generated kernels (libkfuse_bounds.so, built with
KF_BOUNDS from the same sources).  compute-sanitizer is closed on
the GPU pool, so the memory check is our own: every global read of a kernel
must land in one of the launch's external image buffers and every write in the
launch's own output rows, or it is skipped and counted (kf_bounds_report).

Each case asserts zero violations AND that the checked build computes the same
bits as the product library (which test_gpu_parity.py checks against the
oracle).  A self-test (option bounds_shrink: one output row removed from the
writable span) proves the checker reports what it should."""
import importlib.util
import os

import numpy as np
import pytest
import torch

from kf_inputs import gen
from kf_inputs import pipelines as P
from paper_conf_cgo_qiaorht19_b200 import kfuse as K

pytestmark = pytest.mark.gpu
_HERE = os.path.dirname(os.path.abspath(__file__))
_spec = importlib.util.spec_from_file_location("bounds_cases", os.path.join(_HERE, "bounds_cases.py"))
BC = importlib.util.module_from_spec(_spec)
_spec.loader.exec_module(BC)
CASES = BC.cases()


@pytest.fixture(scope="module", autouse=True)
def _precompile_kernels():
    """Compiles this module's kernels (bounds-checking build) up front in parallel
    threads: instant when build() warmed the in-tree cubin cache."""
    from concurrent.futures import ThreadPoolExecutor
    root = os.path.dirname(_HERE)
    spec = importlib.util.spec_from_file_location("warm_test_cache", os.path.join(root, "tools", "warm_test_cache.py"))
    w = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(w)
    jobs = [j for j in w.jobs() if j[3] == "bounds"]
    jobs += [(spec, kind, opts, False) for _, spec, kind, opts in CASES]   # product twins
    with ThreadPoolExecutor(max(1, min(32, os.cpu_count() or 1))) as ex:
        list(ex.map(w.compile_job, jobs))
    yield


@pytest.fixture(scope="module")
def B():
    """A second binding instance bound to the bounds-checking build."""
    spec = importlib.util.spec_from_file_location("kfuse_bounds", K.__file__)
    mod = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mod)
    mod.lib = mod._open(os.path.join(os.path.dirname(K.__file__), "libkfuse_bounds.so"))
    assert "BOUNDS" in mod.version()
    return mod


def _inputs(spec, seed):
    return [gen.image(spec["dtype"], seed + 101 * j, spec["width"], spec["height"]) for j in range(spec["n_inputs"])]


def _plan(mod, spec, kind, opts=None):
    p = mod.Pipeline.from_spec(spec, opts)
    return p.plan_unfused() if kind == "unfused" else p.plan_fusion(kind)


def _alloc(spec, rows=None):
    H, W = rows if rows is not None else spec["height"], spec["width"]
    dt = torch.float32 if spec["dtype"] == "f32" else torch.uint8
    shape = (H, W) if spec["dtype"] == "f32" else (H, W, 4)
    return [torch.full(shape, 7, dtype=dt, device="cuda") for _ in spec["outputs"]]


def _run(plan, spec, ins):
    d_in = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in ins]
    outs = _alloc(spec)
    plan.run(d_in, outs)
    torch.cuda.synchronize()
    return [o.cpu().numpy() for o in outs]


def test_product_library_has_no_bounds_checks():
    p = K.Pipeline.from_spec(P.harris(16, 16))
    with pytest.raises(K.KfError):
        K.bounds_report(p)


@pytest.mark.parametrize("case", CASES, ids=[c[0] for c in CASES])
def test_no_out_of_bounds_access(B, case):
    _, spec, kind, opts = case
    ins = _inputs(spec, 21)
    plan = _plan(B, spec, kind, opts)
    got = _run(plan, spec, ins)
    n, addr, k = B.bounds_report(plan.pipe)
    assert n == 0, f"{n} out-of-bounds accesses, first {'read' if k == 0 else 'write' if k == 1 else 'index'} at {addr:#x}"
    ref = _run(_plan(K, spec, kind, opts), spec, ins)
    for g, r in zip(got, ref):
        np.testing.assert_array_equal(g, r)


@pytest.mark.parametrize("wl", ["harris", "deep10"])
def test_bands_host_and_batch_in_bounds(B, wl):
    """Row bands read exactly their declared input rows [row0 - R, row1 + R) and
    write only their own rows; kf_run_host's staged bands and kf_run_batch's
    overlapping frames stay inside their buffers too."""
    spec = P.WORKLOADS[wl](300, 200)
    ins = _inputs(spec, 5)
    plan = _plan(B, spec, "b200")
    full = _run(plan, spec, ins)[0]
    H, R = spec["height"], plan.halo_rows
    for r0, r1 in [(0, 13), (13, 90), (90, 91), (91, 200)]:
        a0, a1 = max(0, r0 - R), min(H, r1 + R)
        d_in = [torch.from_numpy(np.ascontiguousarray(x[a0:a1])).cuda() for x in ins]
        out = _alloc(spec, r1 - r0)
        plan.run_band(r0, r1, d_in, a0, a1, out)
        torch.cuda.synchronize()
        np.testing.assert_array_equal(out[0].cpu().numpy(), full[r0:r1])
    hout = np.empty_like(full)
    plan.run_host([np.ascontiguousarray(a) for a in ins], [hout])
    np.testing.assert_array_equal(hout, full)
    fin = [[torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in ins] for _ in range(3)]
    fout = [_alloc(spec) for _ in range(3)]
    plan.run_batch(fin, fout)
    torch.cuda.synchronize()
    for f in fout:
        np.testing.assert_array_equal(f[0].cpu().numpy(), full)
    n, addr, k = B.bounds_report(plan.pipe)
    assert n == 0, f"{n} out-of-bounds accesses, first kind {k} at {addr:#x}"


def test_tall_image_bands_in_bounds(B):
    """Many strips and waves (130 x 1030), kf_run_host's 8 bands."""
    for wl in ["harris", "deep10"]:
        spec = P.WORKLOADS[wl](130, 1030)
        ins = _inputs(spec, 6)
        plan = _plan(B, spec, "b200")
        full = _run(plan, spec, ins)[0]
        hout = np.empty_like(full)
        plan.run_host([np.ascontiguousarray(a) for a in ins], [hout])
        np.testing.assert_array_equal(hout, full)
        n, addr, k = B.bounds_report(plan.pipe)
        assert n == 0, f"{wl}: {n} out-of-bounds accesses, first kind {k} at {addr:#x}"


def test_checker_self_test(B):
    """With one output row removed from every launch's writable span, the
    checker must report writes, the first inside that row, and leave exactly
    that row unwritten."""
    spec = P.harris(300, 200)
    ins = _inputs(spec, 3)
    plan = _plan(B, spec, "b200", {"bounds_shrink": 1})
    d_in = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in ins]
    out = _alloc(spec)
    plan.run(d_in, out)
    n, addr, k = B.bounds_report(plan.pipe)
    assert n > 0 and k == 1
    row = (addr - out[0].data_ptr()) // (300 * 4)
    assert row == 199
    got = out[0].cpu().numpy()
    ref = _run(_plan(K, spec, "b200"), spec, ins)[0]
    np.testing.assert_array_equal(got[:199], ref[:199])
    assert np.all(got[199] == 7)
    assert B.bounds_report(plan.pipe)[0] == 0   # the report clears the record

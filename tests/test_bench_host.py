"""Host-side logic of bench.py (CPU): the algorithmic DRAM bytes per pixel it
derives from a plan's blocks must reproduce the SURVEY §8(d) table -- the
numerator of every roofline fraction the bench reports."""
import bench
from kf_inputs import pipelines as P
from paper_conf_cgo_qiaorht19_b200 import kfuse as K


def _plan_bytes(spec, kind):
    p = K.Pipeline.from_spec(spec)
    plan = p.plan_unfused() if kind == "unfused" else p.plan_basic("paper") if kind == "basic" else p.plan_fusion(kind)
    return bench.alg_bytes_per_px(spec, plan.blocks)


def test_alg_bytes_match_survey_table():
    """Harris unfused 84 (R48+W36), paper plan 60, full fusion 8;
    Unsharp unfused 44, fused 8; C4 deep10 unfused 100, paper plan 92, fused 8."""
    h = P.harris(64, 64)
    assert [_plan_bytes(h, k) for k in ("unfused", "paper", "b200")] == [84, 60, 8]
    u = P.unsharp(64, 64)
    assert [_plan_bytes(u, k) for k in ("unfused", "b200")] == [44, 8]
    d = P.deep10(64, 64)
    assert [_plan_bytes(d, k) for k in ("unfused", "paper", "b200")] == [100, 92, 8]


def test_workload_spec_names():
    spec, seed = bench.workload_spec("sobel:2048")
    assert spec["name"] == "sobel" and spec["width"] == spec["height"] == 2048
    spec, seed = bench.workload_spec("C5")
    assert (spec["width"], spec["height"], seed) == (16384, 16384, 5)


def test_host_cpu_reports_cores():
    h = bench.host_cpu()
    assert h["nproc"] and h["nproc"] >= 1

"""C-ABI on CPU (no GPU calls): the library loads and exports every symbol the
header declares; the C++ planner agrees partition-for-partition with the
reference planner (oracle/planner.py); argument validation; generated kernels
compile with NVRTC for sm_100a."""
import os
import random
import re

import pytest

from kf_inputs import pipelines as P
from oracle import planner as PL
from paper_conf_cgo_qiaorht19_b200 import kfuse as K

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_exports_every_declared_symbol():
    with open(os.path.join(ROOT, "include", "kfuse.h")) as f:
        hdr = f.read()
    declared = set(re.findall(r"^\s*(?:[\w\s\*]+?)\b(kf_\w+)\s*\(", hdr, re.M))
    assert len(declared) >= 28
    for name in declared:
        assert hasattr(K.lib, name), f"libkfuse.so does not export {name}"
    assert declared <= set(K.EXPORTED), sorted(declared - set(K.EXPORTED))
    assert "sm_100a" in K.version()


def _ref_model(profile):
    return {"paper": PL.PAPER_PROFILE, "b200": PL.B200_PROFILE, "b200roof": PL.B200_ROOF_PROFILE}[profile]


def _compare(spec, profile):
    ref = PL.get_legal_partitions(spec, _ref_model(profile))
    p = K.Pipeline.from_spec(spec)
    plan = p.plan_fusion(profile)
    assert plan.blocks == ref.blocks
    assert plan.objective == ref.beta
    assert [(c[0], c[1], c[2]) for c in plan.cuts] == [(c[1], c[2], c[3]) for c in ref.cuts]
    for (ks, kd), e in ref.info.items():
        got = plan.edge(ks, kd)
        assert got["w"] == e.w and got["ctx_legal"] == e.ctx_legal and got["profitable"] == e.profitable
        assert got["is_eps"] == (e.weight[1] == 1)
    return plan


@pytest.mark.parametrize("wl", ["harris", "shitomasi", "unsharp", "sobel", "enhance", "deep10", "two_input"])
@pytest.mark.parametrize("profile", ["paper", "b200", "b200roof"])
def test_planner_matches_reference_on_workloads(wl, profile):
    _compare(P.WORKLOADS[wl](64, 64), profile)


@pytest.mark.parametrize("seed", range(30))
def test_roofline_planner_matches_reference_on_random_dags(seed):
    """The ROOFLINE profile (R-20): edge weights, cuts and partition equal the
    independent Python planner's on random DAGs of both dtypes."""
    rng = random.Random(61000 + seed)
    spec = P.random_pipeline(rng, 40, 30, rng.choice(["f32", "u8x4"]), rng.randint(2, 8))
    _compare(spec, "b200roof")


def test_harris_plan_pins_through_the_abi():
    """Fig. 3 through the C-ABI: 6 blocks, beta 912, first cut {sy,gy} at 2 eps after 8 phases."""
    plan = _compare(P.harris(256, 256), "paper")
    assert plan.num_launches == 6 and plan.objective == (912 << 20, 0)
    assert plan.cuts[0] == ([3, 6], (0, 2), 8)
    assert plan.halo_rows == 2


@pytest.mark.parametrize("seed", range(80))
def test_planner_matches_reference_on_random_dags(seed):
    rng = random.Random(5000 + seed)
    spec = P.random_pipeline(rng, 16, 16, rng.choice(["f32", "u8x4"]), rng.randint(1, 9))
    _compare(spec, rng.choice(["paper", "b200"]))


def test_unfused_and_from_blocks():
    spec = P.harris(32, 32)
    p = K.Pipeline.from_spec(spec)
    assert p.plan_unfused().blocks == [[k] for k in range(9)]
    p2 = K.Pipeline.from_spec(spec)
    plan = p2.plan_from_blocks([0, 1, 2, 3, 4, 2, 3, 4, 5])
    assert plan.blocks == [[0], [1], [2, 5], [3, 6], [4, 7], [8]]
    p3 = K.Pipeline.from_spec(spec)
    with pytest.raises(K.KfError) as e:
        p3.plan_from_blocks([0, 0, 1, 2, 3, 4, 5, 6, 7])     # {dx, dy}: two sinks
    assert e.value.name == "KF_ERR_ILLEGAL_BLOCK"
    p4 = K.Pipeline.from_spec(spec)
    with pytest.raises(K.KfError):
        p4.plan_from_blocks([0, 1, 0, 3, 4, 5, 6, 7, 8])     # {dx, sx}: external output (Fig. 2c)
    p5 = K.Pipeline.from_spec(spec)
    assert len(p5.plan_from_blocks([0] * 9).blocks) == 1    # whole DAG is dependence-legal


def test_argument_validation():
    p = K.Pipeline(8, 8, "f32")
    i = p.add_input()
    with pytest.raises(K.KfError) as e:
        p.add_point_op([i + 5], [P.L(0)])
    assert e.value.name == "KF_ERR_BAD_ID"
    with pytest.raises(K.KfError) as e:
        p.add_point_op([i], [P.L(0), P.ADD])
    assert e.value.name == "KF_ERR_PROGRAM"
    with pytest.raises(K.KfError) as e:
        p.add_point_op([i], [P.L(0), P.SHR(1)])              # integer op in a float pipeline
    assert e.value.name == "KF_ERR_PROGRAM"
    with pytest.raises(K.KfError) as e:
        p.add_local_op(i, [[1, 1]], "clamp")                   # even mask
    assert e.value.name == "KF_ERR_MASK"
    a = p.add_local_op(i, [[1, 2, 1]], "mirror")
    p.mark_output(a)
    with pytest.raises(K.KfError):
        p.mark_output(a)
    p.plan_unfused()
    with pytest.raises(K.KfError) as e:
        p.add_point_op([a], [P.L(0)])
    assert e.value.name == "KF_ERR_FROZEN"
    q = K.Pipeline(8, 8, "u8x4")
    j = q.add_input()
    with pytest.raises(K.KfError) as e:
        q.add_local_op(j, [[0.5, 1, 0.5]], "clamp")
    assert e.value.name == "KF_ERR_MASK"
    with pytest.raises(K.KfError):
        q.add_local_op(j, [[1, 1, 1]], "constant", constant=300)
    with pytest.raises(K.KfError):
        K.Pipeline(0, 5, "f32")


def test_run_batch_validates_frames_without_a_gpu():
    """kf_run_batch checks frame disjointness before touching CUDA: an output that
    overlaps another frame's input or output is KF_ERR_ARG; so is a negative count;
    zero frames is a no-op.  (Addresses are never dereferenced on this path.)"""
    spec = P.harris(64, 32)
    plan = K.Pipeline.from_spec(spec).plan_fusion("b200")
    nb = 64 * 32 * 4
    base = 1 << 40
    with pytest.raises(K.KfError) as e:      # frame 1 reads frame 0's output
        plan.run_batch([[base], [base + nb]], [[base + nb], [base + 2 * nb]], stream=0)
    assert e.value.name == "KF_ERR_ARG" and "share memory" in str(e.value)
    with pytest.raises(K.KfError) as e:      # outputs overlap by one pixel
        plan.run_batch([[base], [base]], [[base + nb], [base + 2 * nb - 4]], stream=0)
    assert e.value.name == "KF_ERR_ARG"
    plan.run_batch([], [], stream=0)
    st = K.lib.kf_run_batch(plan.pipe.h, plan.h, -1, K._ptrs([base]), 1, K._ptrs([base + nb]), 1, None)
    assert st != 0


def test_peer_calls_validate_without_a_gpu():
    """The multi-GPU entry points check their arguments before touching CUDA:
    same-device peer enable is a no-op; bad segment counts fail with KF_ERR_ARG."""
    K.peer_enable(0, 0)
    with pytest.raises(K.KfError) as e:
        K.peer_wait([1] * 5, [1] * 5, 8, stream=0)          # more than 4 counters
    assert e.value.name == "KF_ERR_ARG"
    with pytest.raises(K.KfError) as e:
        K.peer_signal([1] * 5, stream=0)
    assert e.value.name == "KF_ERR_ARG"


def test_repeat_mixing_is_not_fused():
    """Reading R-8: a fused block's local kernels all use REPEAT or none does."""
    p = P.Pipeline("mix", 16, 16, "f32")
    i = p.input()
    a = p.local("a", i, P.GAUSS3_N, "repeat")
    b = p.local("b", a, P.GAUSS3_N, "clamp")
    p.output(b)
    spec = p.spec()
    plan = K.Pipeline.from_spec(spec).plan_fusion("b200")
    assert plan.blocks == [[0], [1]]
    with pytest.raises(K.KfError):
        K.Pipeline.from_spec(spec).plan_from_blocks([0, 0])


@pytest.mark.parametrize("seed", range(10))
def test_generated_kernels_compile_for_sm100a(seed, tmp_path, monkeypatch):
    """Every block of random plans compiles with NVRTC to an sm_100a cubin."""
    monkeypatch.setenv("KFUSE_CACHE_DIR", str(tmp_path))
    rng = random.Random(9000 + seed)
    spec = P.random_pipeline(rng, 20, 12, rng.choice(["f32", "u8x4"]), rng.randint(2, 7))
    p = K.Pipeline.from_spec(spec)
    plan = p.plan_fusion(rng.choice(["paper", "b200"]))
    plan.compile()
    cubins = list(tmp_path.glob("*.cubin.z"))   # zlib-compressed cache entries: "KFZ1", u64 size, deflate
    assert len(cubins) == len(plan.blocks)
    import struct
    import zlib
    z = cubins[0].read_bytes()
    assert z[:4] == b"KFZ1"
    blob = zlib.decompress(z[12:])
    assert len(blob) == struct.unpack("<Q", z[4:12])[0]
    assert blob[:4] == b"\x7fELF"


# ----------------------------------------- basic [12] and exact planners (§8(f))


@pytest.mark.parametrize("wl", ["harris", "shitomasi", "unsharp", "sobel", "enhance", "deep10"])
@pytest.mark.parametrize("profile", ["paper", "b200"])
def test_basic_planner_matches_reference(wl, profile):
    spec = P.WORKLOADS[wl](64, 64)
    plan = K.Pipeline.from_spec(spec).plan_basic(profile)
    assert plan.blocks == PL.basic_fusion(spec, _ref_model(profile))


@pytest.mark.parametrize("seed", range(60))
def test_basic_planner_matches_reference_on_random_dags(seed):
    rng = random.Random(8000 + seed)
    spec = P.random_pipeline(rng, 16, 16, rng.choice(["f32", "u8x4"]), rng.randint(1, 9))
    profile = rng.choice(["paper", "b200"])
    plan = K.Pipeline.from_spec(spec).plan_basic(profile)
    assert plan.blocks == PL.basic_fusion(spec, _ref_model(profile))


def _check_exact(spec, profile):
    m = _ref_model(profile)
    plan = K.Pipeline.from_spec(spec).plan_exact(profile)
    best, _ = PL.brute_force(spec, m)
    assert plan.objective == best
    g = PL.graph(spec)
    info = PL.edge_weights(g, m)
    assert sorted(k for b in plan.blocks for k in b) == list(range(g.n))
    for b in plan.blocks:
        assert PL.is_legal(g, set(b), m, info)
    assert K.Pipeline.from_spec(spec).plan_fusion(profile).objective <= plan.objective
    return plan


@pytest.mark.parametrize("wl", ["harris", "shitomasi", "unsharp", "sobel", "enhance", "deep10"])
@pytest.mark.parametrize("profile", ["paper", "b200"])
def test_exact_planner_equals_bruteforce_on_workloads(wl, profile):
    _check_exact(P.WORKLOADS[wl](64, 64), profile)


@pytest.mark.parametrize("seed", range(50))
def test_exact_planner_equals_bruteforce_on_random_dags(seed):
    rng = random.Random(9000 + seed)
    spec = P.random_pipeline(rng, 16, 16, rng.choice(["f32", "u8x4"]), rng.randint(1, 8))
    _check_exact(spec, rng.choice(["paper", "b200"]))


@pytest.mark.parametrize("seed", range(20))
def test_exact_planner_equals_bruteforce_roofline(seed):
    """kf_plan_exact under the ROOFLINE weights (R-20) = the brute-force optimum of
    the independent Python planner, and Alg. 1 never beats it."""
    rng = random.Random(9700 + seed)
    spec = P.random_pipeline(rng, 16, 16, rng.choice(["f32", "u8x4"]), rng.randint(1, 7))
    _check_exact(spec, "b200roof")


def test_exact_planner_beats_min_cut_counterexample():
    """Alg. 1 reaches 350 on the 5-local chain, the optimum is 550."""
    p = P.Pipeline("chain", 32, 32, "f32")
    x = p.input()
    for k, n_alu in enumerate([12, 8, 4, 2, 1]):
        x = p.local(f"l{k}", x, [[1] * 3] * 3, "clamp", cost=(n_alu, 0))
    p.output(x)
    over = dict(ts=1.0, c_alu=1.0, c_mshared=2.0)
    pipe = K.Pipeline.from_spec(p.spec())
    assert pipe.plan_fusion("paper", **over).objective == (350 << 20, 0)
    assert K.Pipeline.from_spec(p.spec()).plan_exact("paper", **over).objective == (550 << 20, 0)


def test_exact_planner_size_limit():
    p = P.Pipeline("long", 16, 16, "f32")
    x = p.input()
    for k in range(17):
        x = p.point(f"p{k}", [x], [("LOAD", 0, 0), ("CONST", 0, 1.0), ("ADD", 0, 0)])
    p.output(x)
    with pytest.raises(K.KfError):
        K.Pipeline.from_spec(p.spec()).plan_exact("paper")


def test_swar_form_chosen_by_interval_analysis():
    """u8x4 codegen: kernels whose lanes provably fit 16 bits run
    two channels per op (PRMT-unpacked SWAR); a 16-bit-overflowing mask, ABS, DIV,
    SELECT and a variable product fall back to per-channel int32; option swar=0
    turns the form off."""
    spec = P.swar_stress(64, 48)
    plan = K.Pipeline.from_spec(spec).plan_unfused()
    form = {}
    for b in range(plan.num_launches):
        body = plan.source(b).split("_fast_di(")[1]
        form[spec["ops"][b]["name"]] = "swar" if "__byte_perm" in body else "int32"
    assert form == {"a": "swar", "b": "swar", "c": "swar", "d": "swar", "e": "int32", "f": "int32",
                    "g": "int32", "h": "int32", "k": "int32", "m": "swar"}
    plan = K.Pipeline.from_spec(spec, {"swar": 0}).plan_unfused()
    assert all("__byte_perm" not in plan.source(b).split("_fast_di(")[1] for b in range(plan.num_launches))
    c4, _ = P.config("C4")
    src = K.Pipeline.from_spec(c4).plan_fusion("b200").source(0).split("_fast_di(")[1]
    assert "kf_unpack" not in src and "kf_lut(" not in src   # all ten deep10 kernels in SWAR form


def _di(src: str) -> str:
    """The interior variant of a generated block (the hot loop's function)."""
    body = src.split("_fast_di(")[1]
    return body[:body.index("\n}\n")]


def test_rolled_u8x4_codegen_choices():
    """What the code generator decides for deep10 (C4, a rolled u8x4 body), read
    from the generated source: the warm-up rows run in a
    loop of their own and the steady-state loop carries no guards (warm_skip=2);
    warm_skip=1 puts warp-uniform guards into the one loop; the LUT is gathered
    from a shared-memory copy; the input and k0 keep their far rows in
    shared-memory delay lines, which frees the registers for k4's unpacked ring;
    f32 pipelines and option delay_smem=0 get none."""
    c4, _ = P.config("C4")
    src = K.Pipeline.from_spec(c4).plan_fusion("b200").source(0)
    di = _di(src)
    assert "for (; u < min(nit, 12); u += 1)" in di and "for (; u < nit; u += 1)" in di
    steady = di[di.index("for (; u < nit; u += 1)"):]
    assert "if (u + 0 >= " not in steady
    assert "__shared__ int kf_lutsh_0_6[256];" in src and "kf_lutsh_0_6[KF_IDX(" in di
    assert "uint4 *dl0 = " in di and "uint4 *dl1 = " in di                  # input and k0 delay lines
    assert "- 6) & 7) * 32]" in di and "- 4) & 7) * 32]" in di              # ages 6 and 4 read from them
    assert "live~152" in src.splitlines()[0]
    guarded = _di(K.Pipeline.from_spec(c4, {"warm_skip": 1}).plan_fusion("b200").source(0))
    assert "for (; u < min(nit," not in guarded and "if (u + 0 >= 12) {" in guarded
    no_dl = K.Pipeline.from_spec(c4, {"delay_smem": 0}).plan_fusion("b200").source(0)
    assert "uint4 *dl" not in no_dl and "live~164" in no_dl.splitlines()[0]
    no_lut = K.Pipeline.from_spec(c4, {"lut_smem": 0}).plan_fusion("b200").source(0)
    assert "kf_lutsh_" not in no_lut and "__ldg(kf_lut_0_6 + KF_IDX(" in no_lut
    f32 = K.Pipeline.from_spec(P.enhance(2048, 2048)).plan_fusion("b200").source(0)
    assert "rolled" in f32.splitlines()[0] and "uint4 *dl" not in f32


def test_shared_luts_fit_static_shared_memory():
    """Shared-memory table copies are dropped when rings x warps per CTA plus the
    tables would exceed 48 KB of static shared memory (found by the fuzz: a LUT
    under cta_warps=4)."""
    c4, _ = P.config("C4")
    one = K.Pipeline.from_spec(c4).plan_fusion("b200").source(0)
    assert "kf_lutsh_" in one
    many = K.Pipeline.from_spec(c4, {"cta_warps": 8}).plan_fusion("b200").source(0)
    m = re.search(r"_smem\[(\d+)\]", many)
    assert m and int(m.group(1)) + (1024 if "kf_lutsh_" in many else 0) <= 49152


def test_schedule_options_api():
    """kf_set_option / kf_get_option: known options with defaults and ranges; unknown
    names, out-of-range values and the test-only / experimental options are
    rejected by the product library (no environment variable reaches it)."""
    p = K.Pipeline(64, 32)
    assert p.get_option("smem_rows") == 12 and p.get_option("swar") == 1
    p.set_option("smem_rows", 6)
    assert p.get_option("smem_rows") == 6
    for bad in ("naive_border", "v8", "persist", "nlong", "no_such_option", "KFUSE_SWAR"):
        with pytest.raises(K.KfError) as e:
            p.set_option(bad, 1)
        assert e.value.name == "KF_ERR_ARG"
    with pytest.raises(K.KfError):
        p.set_option("smem_rows", 1000)
    assert "TEST HOOKS" not in K.version()


def test_library_reads_no_environment():
    """The product library's only getenv is the cubin cache directory: no knob can
    change what kf_run computes."""
    import subprocess
    so = os.path.join(os.path.dirname(K.__file__), "libkfuse.so")
    syms = subprocess.run(["nm", "-D", "--undefined-only", so], capture_output=True, text=True).stdout
    strings = subprocess.run(["strings", so], capture_output=True, text=True).stdout.split()
    assert "KFUSE_CACHE_DIR" in strings
    assert not [t for t in strings if t.startswith("KFUSE_") and t != "KFUSE_CACHE_DIR"], \
        [t for t in strings if t.startswith("KFUSE_")]
    assert "getenv" in syms


def test_staged_profile_reductions_through_the_abi():
    """The product planner's STAGED factor (R-4) reduces to the paper's Eq. 7 at a
    1x1 tile (Harris 328 / 256) and to no recompute at an
    unbounded tile (400 - 8 = 392)."""
    spec = P.harris(64, 64)
    ix = {o["name"]: k for k, o in enumerate(spec["ops"])}
    one = K.Pipeline.from_spec(spec).plan_fusion(K.model_params("b200", tile_w=1, tile_h=1))
    assert one.edge(ix["sx"], ix["gx"])["w"] == 328.0 and one.edge(ix["sxy"], ix["gxy"])["w"] == 256.0
    big = K.Pipeline.from_spec(spec).plan_fusion(K.model_params("b200", tile_w=1 << 20, tile_h=1 << 20))
    assert abs(big.edge(ix["sx"], ix["gx"])["w"] - 392.0) < 1e-3


def _build_c_example(tmp_path):
    import subprocess
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    libdir = os.path.join(root, "paper_conf_cgo_qiaorht19_b200")
    exe = str(tmp_path / "harris_c")
    subprocess.run(["gcc", "-std=c99", "-Wall", "-Wextra", "-Werror", "-I", os.path.join(root, "include"),
                    os.path.join(root, "examples", "harris_c.c"), "-L", libdir, "-lkfuse",
                    f"-Wl,-rpath,{libdir}", "-o", exe], check=True)
    return exe


def test_c_abi_from_plain_c(tmp_path):
    """include/kfuse.h compiles as C99 (-Wall -Wextra -Werror) and the library is
    usable from plain C: examples/harris_c.c builds the Harris DAG, and Alg. 1
    under the paper profile reproduces Fig. 3 (6 blocks, beta 912) and the B200
    profile one fused launch."""
    import subprocess
    out = subprocess.run([_build_c_example(tmp_path)], capture_output=True, text=True, check=True).stdout
    assert "paper profile: 6 blocks, beta = 912.0" in out
    assert "b200 profile: 1 block(s), 1 launch(es), halo rows 2" in out

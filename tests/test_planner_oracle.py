"""Pins for the reference planner (oracle/planner.py) against the paper's worked
Harris example (Fig. 3), its application statements (§V) and
textbook reductions (brute-force min cut, brute-force optimum of Eq. 1).  CPU only."""
import random

import pytest

from kf_inputs import pipelines as P
from oracle import planner as PL

EPS = (0, 1)
FIX = PL.FIX


def names(spec, ks):
    return [spec["ops"][k]["name"] for k in ks]


@pytest.fixture(scope="module")
def harris():
    return P.harris(64, 64)


def test_harris_edge_weights(harris):
    """(sx,gx)=(sy,gy)=328, (sxy,gxy)=256, the other seven edges eps
    (tg=400, cALU=4, nALU=2, sz=9, IS = number of input images, gamma omitted)."""
    pl = PL.get_legal_partitions(harris)
    w = {tuple(names(harris, k)): e.weight for k, e in pl.info.items()}
    assert len(w) == 10
    assert w[("sx", "gx")] == (328 * FIX, 0) and w[("sy", "gy")] == (328 * FIX, 0)
    assert w[("sxy", "gxy")] == (256 * FIX, 0)
    assert sum(1 for v in w.values() if v == EPS) == 7


def test_harris_legality_statements(harris):
    """(dx,sx) illegal: external output; (gx,hc) illegal: external
    inputs; whole DAG dependence-legal but fails Eq. 2 with
    five smem kernels vs cMshared = 2."""
    g = PL.graph(harris)
    m = PL.PAPER_PROFILE
    idx = {o["name"]: k for k, o in enumerate(harris["ops"])}
    assert not PL._dependence_legal(g, {idx["dx"], idx["sx"]})
    assert not PL._dependence_legal(g, {idx["gx"], idx["hc"]})
    everything = set(range(9))
    assert PL._dependence_legal(g, everything)
    assert not PL._resource_legal(g, everything, m)
    assert PL._resource_legal(g, everything, PL.Model(c_mshared=5.0))
    assert not PL._resource_legal(g, everything, PL.Model(c_mshared=4.99))


def test_harris_fig3_cut_sequence(harris):
    """Fig. 3a: starting from dx, after eight min-cut phases the global minimum cut
    has weight 2 eps and separates {sy, gy}; the remaining block
    is illegal via dy -> sy; the panel edge counts after each
    cut are 8, 7, 5, 4, 3 (Fig. 3b-f token counts)."""
    pl = PL.get_legal_partitions(harris)
    first = pl.cuts[0]
    assert first[3] == 8 and first[2] == (0, 2)
    assert names(harris, first[1]) == ["sy", "gy"]
    rest = sorted(set(range(9)) - set(first[1]))
    g = PL.graph(harris)
    assert not PL._dependence_legal(g, set(rest))
    remaining = []
    cut_edges = set()
    for blk, side, w, ph in pl.cuts:
        other = set(blk) - set(side)
        for (a, b) in pl.info:
            if (a in side and b in other) or (b in side and a in other):
                cut_edges.add((a, b))
        remaining.append(10 - len(cut_edges))
    assert remaining == [8, 7, 5, 4, 3]


def test_harris_final_plan_and_beta(harris):
    """Final partition {dx},{dy},{sx,gx},{sy,gy},{sxy,gxy},{hc}, beta = 912, which is
    also the brute-force optimum of Eq. 1."""
    pl = PL.get_legal_partitions(harris)
    blocks = sorted(tuple(names(harris, b)) for b in pl.blocks)
    assert blocks == sorted([("dx",), ("dy",), ("sx", "gx"), ("sy", "gy"), ("sxy", "gxy"), ("hc",)])
    assert pl.beta == (912 * FIX, 0)
    best, _ = PL.brute_force(harris)
    assert best == pl.beta


def test_harris_b200_profile_fuses_whole(harris):
    """With cMshared >= 5 the whole DAG is legal (five smem kernels)."""
    pl = PL.get_legal_partitions(harris, PL.B200_PROFILE)
    assert pl.blocks == [list(range(9))]
    assert pl.beta[1] == 7   # seven context-illegal edges stay eps inside the block


def test_eq9_fused_mask_sizes():
    """Eq. 9 examples: 3x3 (+) 5x5 -> 7x7 = 49; 3x3 (+) 3x3 -> 5x5 = 25."""
    for ms, md, g_expect in [(3, 5, 49), (3, 3, 25), (5, 3, 49), (5, 5, 81)]:
        p = P.Pipeline("ll", 32, 32, "f32")
        i = p.input()
        a = p.local("a", i, [[1] * ms] * ms, "clamp", cost=(1, 0))
        b = p.local("b", a, [[1] * md] * md, "clamp")
        p.output(b)
        g = PL.graph(p.spec())
        m = PL.Model(ts=1.0, c_alu=1.0)
        sc, w = PL.benefit(g, 0, 1, m)
        assert sc == "l2l" and w == 400.0 - g_expect


def test_point_to_local_eq8():
    """Eq. 8: w = tg - costop * IS_ks * sz(kd), costop = cALU nALU + cSFU nSFU (Eq. 6)."""
    p = P.Pipeline("pl", 32, 32, "f32")
    i, j = p.input(), p.input()
    a = p.point("a", [i, j], [P.L(0), P.L(1), P.ADD, P.SQRT])
    b = p.local("b", a, [[1] * 5] * 5, "clamp")
    p.output(b)
    g = PL.graph(p.spec())
    assert g.cost[0] == (1, 1)
    sc, w = PL.benefit(g, 0, 1, PL.PAPER_PROFILE)
    assert sc == "p2l" and w == 400.0 - (4 * 1 + 16 * 1) * 2 * 25


def test_unsharp_fused_whole():
    """Unsharp: blur + three point kernels all reading the input (Fig. 2b shared input)
    is fused into one kernel by the optimized method."""
    pl = PL.get_legal_partitions(P.unsharp(64, 64))
    assert pl.blocks == [[0, 1, 2, 3]]


def test_enhance_chain_fused_whole():
    """Enhancement chain fully fused."""
    s = P.enhance(64, 64)
    assert PL.get_legal_partitions(s).blocks == [list(range(len(s["ops"])))]


def test_sobel_fused_whole():
    """Sobel dx, dy -> magnitude: fused by the optimized method."""
    assert PL.get_legal_partitions(P.sobel(64, 64)).blocks == [[0, 1, 2]]


def test_night_unprofitable_local_to_local():
    """Night: Atrous0 (3x3) -> Atrous1 (5x5, 68 ALU ops) -> Scoto (point, 89 ALU ops);
    only Atrous1 + Scoto are fused, the local-to-local pair is too costly
    (PAPER.md:1436-1506).  Benefit <= 0 makes any block containing it illegal (:500-505)."""
    p = P.Pipeline("night", 64, 64, "f32")
    i = p.input()
    a0 = p.local("atrous0", i, [[1] * 3] * 3, "clamp", cost=(17, 0))
    a1 = p.local("atrous1", a0, [[1] * 5] * 5, "clamp", cost=(68, 0))
    sc = p.point("scoto", [a1], [P.L(0)], cost=(89, 0))
    p.output(sc)
    pl = PL.get_legal_partitions(p.spec())
    assert sorted(pl.blocks) == [[0], [1, 2]]
    assert not pl.info[(0, 1)].profitable


def test_all_point_graph_fused_in_first_iteration():
    """'if all the kernels are point operators ... the whole graph would be fused into
    one kernel' at the beginning."""
    p = P.Pipeline("pts", 16, 16, "f32")
    i = p.input()
    a = p.point("a", [i], [P.L(0), P.C(2), P.MUL])
    b = p.point("b", [i, a], [P.L(0), P.L(1), P.ADD])
    c = p.point("c", [a, b], [P.L(0), P.L(1), P.MUL])
    p.output(c)
    pl = PL.get_legal_partitions(p.spec())
    assert pl.blocks == [[0, 1, 2]] and pl.cuts == []


def test_deep10_plans():
    """C4: paper profile fuses only {k5,k6}; the edges k1->k2, k1->k3, k4->k5
    are unprofitable (5x5 per-tap recompute); the B200 (staged) profile fuses all ten."""
    s = P.deep10(64, 64)
    pl = PL.get_legal_partitions(s)
    multi = [b for b in pl.blocks if len(b) > 1]
    assert multi == [[5, 6]]
    unprof = sorted(k for k, e in pl.info.items() if not e.profitable)
    assert unprof == [(1, 2), (1, 3), (4, 5)]
    assert PL.get_legal_partitions(s, PL.B200_PROFILE).blocks == [list(range(10))]


def test_min_cut_suboptimal_counterexample():
    """The recursive min cut is a heuristic for the NP-complete k-cut:
    a 5-local chain with weights 100/200/300/350 and cMshared=2 yields beta 350 while
    the optimum is 550 -- so tests assert beta_plan <= beta*."""
    p = P.Pipeline("chain", 32, 32, "f32")
    x = p.input()
    for k, n_alu in enumerate([12, 8, 4, 2, 1]):
        x = p.local(f"l{k}", x, [[1] * 3] * 3, "clamp", cost=(n_alu, 0))
    p.output(x)
    m = PL.Model(ts=1.0, c_alu=1.0, c_mshared=2.0)
    pl = PL.get_legal_partitions(p.spec(), m)
    best, _ = PL.brute_force(p.spec(), m)
    assert pl.beta == (350 * FIX, 0) and best == (550 * FIX, 0)


@pytest.mark.parametrize("seed", range(40))
def test_stoer_wagner_equals_bruteforce_min_cut(seed):
    """Stoer-Wagner returns a global minimum cut (textbook reduction: min over all
    bipartitions, [14])."""
    rng = random.Random(seed)
    s = P.random_pipeline(rng, 16, 16, rng.choice(["f32", "u8x4"]), rng.randint(2, 8))
    g = PL.graph(s)
    info = PL.edge_weights(g, PL.PAPER_PROFILE)
    verts = list(range(g.n))
    if len(verts) < 2:
        return
    side, rest, w, phases = PL.stoer_wagner(g, verts, info)
    assert phases == len(verts) - 1
    assert side and rest
    assert w == PL.min_cut_brute(g, verts, info)


@pytest.mark.parametrize("seed", range(60))
def test_plan_is_legal_cover_and_bounded_by_bruteforce(seed):
    """Alg. 1 output: legal, pairwise disjoint, covering and
    beta_plan <= beta* (exhaustive optimum)."""
    rng = random.Random(1000 + seed)
    s = P.random_pipeline(rng, 16, 16, rng.choice(["f32", "u8x4"]), rng.randint(2, 7))
    m = rng.choice([PL.PAPER_PROFILE, PL.B200_PROFILE, PL.Model(c_mshared=3.0, phi_mode=1)])
    pl = PL.get_legal_partitions(s, m)
    g = PL.graph(s)
    seen = sorted(k for b in pl.blocks for k in b)
    assert seen == list(range(g.n))
    for b in pl.blocks:
        assert PL.is_legal(g, set(b), m, pl.info)
    best, _ = PL.brute_force(s, m)
    assert pl.beta <= best
    assert pl.beta[0] <= best[0]


@pytest.mark.parametrize("wl", ["harris", "shitomasi", "unsharp", "sobel", "enhance"])
@pytest.mark.parametrize("prof", ["paper", "b200"])
def test_paper_dags_reach_bruteforce_optimum(wl, prof):
    s = P.WORKLOADS[wl](64, 64)
    m = PL.PAPER_PROFILE if prof == "paper" else PL.B200_PROFILE
    assert PL.get_legal_partitions(s, m).beta == PL.brute_force(s, m)[0]


def test_deep10_reaches_bruteforce_optimum():
    """C4 (10 kernels, Bell(10) partitions): the planner reaches the optimum's real
    part; the exhaustive optimum may hold extra eps terms."""
    s = P.deep10(64, 64)
    for m in (PL.PAPER_PROFILE, PL.B200_PROFILE):
        got, best = PL.get_legal_partitions(s, m).beta, PL.brute_force(s, m)[0]
        assert got[0] == best[0] and got <= best


# ------------------------------------------------ basic fusion [12] (§8(f)3)


@pytest.mark.parametrize("prof", [PL.PAPER_PROFILE, PL.B200_PROFILE])
def test_basic_fusion_paper_statements(prof):
    """PAPER.md:1414-1425 (Table I discussion): the basic fusion of [12] gains most
    on Enhance (a local and two point operators, fully fused); it "failed in
    optimizing" Sobel (local-to-local) and Unsharp (shared input); on Harris and
    ShiTomasi it detects the point-to-local scenarios (the three square ->
    Gaussian pairs of Fig. 3)."""
    e = P.enhance(64, 64)
    assert PL.basic_fusion(e, prof) == [list(range(len(e["ops"])))]
    for wl in ("sobel", "unsharp"):
        s = P.WORKLOADS[wl](64, 64)
        assert PL.basic_fusion(s, prof) == [[k] for k in range(len(s["ops"]))]
    for wl in ("harris", "shitomasi"):
        s = P.WORKLOADS[wl](64, 64)
        multi = [names(s, b) for b in PL.basic_fusion(s, prof) if len(b) > 1]
        assert sorted(multi) == [["sx", "gx"], ["sxy", "gxy"], ["sy", "gy"]]


def test_basic_rules_negative_controls():
    """Hand-built two-kernel blocks: point-to-local and local-to-point are basic-legal,
    local-to-local and a shared input are not."""
    p = P.Pipeline("ctl", 32, 32, "f32")
    x = p.input()
    a = p.point("a", [x], [("LOAD", 0, 0), ("CONST", 0, 2.0), ("MUL", 0, 0)])
    b = p.local("b", a, [[1, 2, 1], [2, 4, 2], [1, 2, 1]], "clamp")
    c = p.local("c", b, [[1, 2, 1], [2, 4, 2], [1, 2, 1]], "clamp")
    d = p.point("d", [c, x], [("LOAD", 0, 0), ("LOAD", 1, 0), ("ADD", 0, 0)])
    p.output(d)
    s = p.spec()
    g = PL.graph(s)
    m = PL.Model(c_mshared=5.0, phi_mode=1)
    info = PL.edge_weights(g, m)
    assert PL.is_legal(g, {0, 1}, m, info) and PL.basic_legal(g, {0, 1}, m, info)        # point-to-local
    assert PL.is_legal(g, {1, 2}, m, info) and not PL.basic_legal(g, {1, 2}, m, info)    # local-to-local
    assert not PL.is_legal(g, {2, 3}, m, info)          # d reads x, the source c does not: Fig. 2d
    assert not PL.basic_legal(g, {0, 1, 2}, m, info)   # local-to-local behind a point
    q = P.Pipeline("shared", 32, 32, "f32")            # Fig. 2b: the shared input
    x = q.input()
    a = q.point("a", [x], [("LOAD", 0, 0), ("CONST", 0, 2.0), ("MUL", 0, 0)])
    e = q.point("e", [a, x], [("LOAD", 0, 0), ("LOAD", 1, 0), ("SUB", 0, 0)])
    q.output(e)
    g = PL.graph(q.spec())
    info = PL.edge_weights(g, m)
    assert PL.is_legal(g, {0, 1}, m, info) and not PL.basic_legal(g, {0, 1}, m, info)


@pytest.mark.parametrize("seed", range(40))
def test_basic_fusion_is_legal_cover_below_optimum(seed):
    """Every basic block is basic-legal (hence IsLegal), the blocks partition the
    kernels, and beta_basic <= beta* (the exhaustive optimum)."""
    rng = random.Random(7000 + seed)
    s = P.random_pipeline(rng, 16, 16, rng.choice(["f32", "u8x4"]), rng.randint(2, 7))
    m = rng.choice([PL.PAPER_PROFILE, PL.B200_PROFILE])
    blocks = PL.basic_fusion(s, m)
    g = PL.graph(s)
    info = PL.edge_weights(g, m)
    assert sorted(k for b in blocks for k in b) == list(range(g.n))
    beta = (0, 0)
    for b in blocks:
        assert PL.basic_legal(g, set(b), m, info)
        beta = PL._add(beta, PL.block_weight(set(b), info))
    assert beta <= PL.brute_force(s, m)[0]


# ------------------------------------------------ ROOFLINE extension (R-20)

def _chain(prog1, prog2, local2=None, dtype="f32"):
    p = P.Pipeline("chain", 64, 64, dtype)
    i = p.input()
    a = p.point("a", [i], prog1)
    b = p.local("b", a, local2, "clamp") if local2 else p.point("b", [a], prog2)
    p.output(b)
    return p.spec()


def test_roofline_memory_bound_pair_saves_the_intermediate_image():
    """Two cheap point kernels: each moves 8 B/px unfused, the fused pair 8 B/px,
    so the benefit is exactly the intermediate's write + read, 2 * 4 B / bw
    (for any overlap: the issue slots of the pair are the sum of its kernels')."""
    m = PL.B200_ROOF_PROFILE
    s = _chain([P.L(0), P.C(1.0), P.ADD], [P.L(0), P.C(2.0), P.MUL])
    info = PL.edge_weights(PL.graph(s), m)
    # overlap 1: T = M + C, and the pair's issue slots are the sum of its kernels'
    assert info[(0, 1)].w == pytest.approx(8.0 / m.bw_bytes_clk, rel=1e-12)
    assert info[(0, 1)].profitable


def test_roofline_issue_bound_pair_gains_nothing():
    """Two POW-heavy point kernels, each issue-bound alone, under a pure roofline
    (overlap 0): fusing saves DRAM time that was hidden anyway, so w = 0 --
    unprofitable, an eps edge (Eq. 12, R-3)."""
    m = PL.Model(**{**PL.B200_ROOF_PROFILE.__dict__, "overlap": 0.0})
    heavy = [P.L(0), P.C(0.5), P.POW, P.C(0.7), P.POW, P.C(0.9), P.POW]
    s = _chain(heavy, heavy)
    g = PL.graph(s)
    assert PL.roofline_time(g, [0], m) > 4 * 2 / m.bw_bytes_clk      # issue-bound alone
    info = PL.edge_weights(g, m)
    assert info[(0, 1)].w == pytest.approx(0.0, abs=1e-12) and not info[(0, 1)].profitable
    assert info[(0, 1)].weight == (0, 1)


def test_roofline_issue_bound_producer_recompute_costs_its_halo():
    """An issue-bound producer feeding a 3x3 local kernel is recomputed on the
    staged halo: the pair costs I(producer) * (tw+2)(th+2)/(tw th) + I(consumer)
    issue slots, which outweighs the consumer's hidden DRAM time when the
    producer is heavy enough -> w < 0, unprofitable."""
    m = PL.B200_ROOF_PROFILE
    heavy = [P.L(0)] + [t for _ in range(15) for t in (P.C(0.99), P.POW)]   # 15 POW: ~600 issue slots / px
    s = _chain(heavy, None, local2=[[1, 1, 1]] * 3)
    m = PL.Model(**{**m.__dict__, "overlap": 0.0})     # a pure roofline for this limit case
    g = PL.graph(s)
    i0 = 15 * 80.0                                     # 15 POW, 80 issue slots each (kfuse.h)
    fac = (m.tile_w + 2) * (m.tile_h + 2) / (m.tile_w * m.tile_h)
    t0, t1 = PL.roofline_time(g, [0], m), PL.roofline_time(g, [1], m)
    w = PL.edge_weights(g, m)[(0, 1)].w
    # the consumer alone is memory-bound (9 taps), the fused pair issue-bound
    assert t1 == pytest.approx(8.0 / m.bw_bytes_clk)
    assert t0 == pytest.approx(i0 / m.issue_lanes_clk)
    assert w == pytest.approx(t0 + t1 - (i0 * fac + 9) / m.issue_lanes_clk, rel=1e-12)
    assert w < 0 and not PL.edge_weights(g, m)[(0, 1)].profitable


@pytest.mark.parametrize("seed", range(25))
def test_roofline_plan_bounded_by_bruteforce(seed):
    """Alg. 1 under the ROOFLINE weights: legal cover, beta <= the exhaustive optimum."""
    rng = random.Random(5100 + seed)
    s = P.random_pipeline(rng, 16, 16, rng.choice(["f32", "u8x4"]), rng.randint(2, 7))
    m = PL.B200_ROOF_PROFILE
    pl = PL.get_legal_partitions(s, m)
    g = PL.graph(s)
    assert sorted(k for b in pl.blocks for k in b) == list(range(g.n))
    for b in pl.blocks:
        assert PL.is_legal(g, set(b), m, pl.info)
    assert pl.beta <= PL.brute_force(s, m)[0]


# --------------------------------- STAGED recompute factor (R-4) reductions

def _staged(tile):
    return PL.Model(c_mshared=5.0, phi_mode=1, tile_w=tile, tile_h=tile)


def test_staged_factor_one_pixel_tile_is_the_papers_per_tap_recompute(harris):
    """R-4 reduces to the paper: with a 1x1 staged tile every consumer pixel
    recomputes its producer on the whole mask footprint, (1+2rx)(1+2ry) = sz(kd),
    i.e. Eq. 7 -- so the point-to-local Harris weights become the worked
    example's 328 / 256."""
    pl = PL.get_legal_partitions(harris, _staged(1))
    w = {tuple(names(harris, k)): e.w for k, e in pl.info.items()}
    assert w[("sx", "gx")] == 328.0 and w[("sy", "gy")] == 328.0 and w[("sxy", "gxy")] == 256.0


def test_staged_factor_infinite_tile_recomputes_nothing(harris):
    """The other end of R-4: as the staged tile grows, the halo share vanishes and
    the producer is computed once per pixel, phi -> costop * IS_ks:
    w(sx, gx) -> tg - cALU*nALU*1 = 400 - 8 = 392, w(sxy, gxy) -> 400 - 16 = 384."""
    pl = PL.get_legal_partitions(harris, _staged(1 << 20))
    w = {tuple(names(harris, k)): e.w for k, e in pl.info.items()}
    assert w[("sx", "gx")] == pytest.approx(392.0, abs=1e-3)
    assert w[("sxy", "gxy")] == pytest.approx(384.0, abs=1e-3)

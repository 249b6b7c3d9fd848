"""TEST INFRASTRUCTURE ONLY -- reference fusion planner, written step by step
from the paper (Qiao et al., CGO'19, §II-§III), plus a brute-force optimum.

Only tests/ (and bench.py's diagnostics) may import this module; the product
planner (paper_conf_cgo_qiaorht19_b200/csrc/planner.cpp) shares no code with it.

Contents, each in the paper's notation:
  kernel_costs()  nALU / nSFU per kernel (SURVEY O1-d reading: explicit cost, else
                  an opcode count)
  edge_weights()  scenario per edge and w_e (Eqs. 3-12)
  is_legal()      dependence (Fig. 2), resources (Eq. 2,
                  PAPER.md:296-321), header, profitability
                    -- readings O1-f/g/h/l
  stoer_wagner()  global min cut, deterministic tie-breaks O1-j ([14])
  get_legal_partitions()  Alg. 1
  brute_force()   exact maximum of Eq. 1 over all partitions into legal blocks
                  (the paper's "exhaustive search")
  basic_fusion()  the "basic" fusion of the authors' previous work [12], the
                  comparison column of Table I,
                  reading R-18

What pins what (R-4, R-7, R-20): the point-based / point-to-local
weights (328/256/eps) and the Eq. 9 sizes are the paper's
numbers; the B200 profile's STAGED recompute factor (R-4) is pinned by its two
reductions (a 1x1 tile gives Eq. 7 and the paper's 328/256; an unbounded tile
gives no recompute); the ROOFLINE weights (R-20) by their limit cases.  Parity
unpinned: the VALUE of the local-to-local locality gain of Eq. 3 (garbled, read
as IS*tg/ts, R-7) -- the paper gives no number for it, only the sign in the
Night filter (an unprofitable local-to-local pair), which
is pinned.

Weights are lexicographic pairs (real, eps-count) with the real part in fixed
point q = floor(w * 2^20 + 0.5) (reading O1-i): sums are exact, so ties
("the first one encountered") are decided identically here
and in the C++ planner.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

SFU_OPS = {"SQRT", "EXP", "LOG", "POW"}
NONARITH = {"LOAD", "CONST"}
FIX = 1 << 20


@dataclass
class Model:
    """Hardware-model constants."""
    tg: float = 400.0       # global-memory access, cycles
    ts: float = 4.0         # shared-memory access, "a few cycles"
    c_alu: float = 4.0
    c_sfu: float = 16.0     # not given; reading O1-b
    gamma: float = 0.0      # omitted in the example
    c_mshared: float = 2.0
    phi_mode: int = 0       # 0 = PAPER (per-tap recompute), 1 = STAGED (O1-g B200 profile)
    tile_w: int = 32
    tile_h: int = 32
    eq3_mode: int = 0       # 0: IS*tg/ts as printed; 1: IS*(tg-ts)  (O1-a)
    bw_bytes_clk: float = 0.0      # phi_mode 2 (ROOFLINE, R-20) only
    issue_lanes_clk: float = 0.0
    overlap: float = 0.0


PAPER_PROFILE = Model()
B200_PROFILE = Model(c_mshared=5.0, phi_mode=1)
# the B200 issue-rate extension (R-20; constants of kfuse.h
# kf_model_params_b200_roofline, restated)
B200_ROOF_PROFILE = Model(c_mshared=5.0, phi_mode=2, tile_w=120, tile_h=32,
                          bw_bytes_clk=22.45, issue_lanes_clk=115.0, overlap=1.0)
# issue slots per pixel of an op-IR opcode (restated from include/kfuse.h, phi_mode 2)
ISSUE_SLOTS = {"LOAD": 0, "CONST": 0, "POW": 80, "LOG": 30, "EXP": 25, "SQRT": 2, "DIV": 15}


@dataclass
class Graph:
    n: int                       # kernels
    kind: list                   # "point" / "local"
    inputs: list                 # image ids per kernel
    n_inputs: int
    rx: list
    ry: list
    mode: list
    outputs: set
    bpp: int
    cost: list                   # (n_alu, n_sfu)
    u8: bool = False             # u8x4 pipeline
    progs: list = field(default_factory=list)   # point body / local post program per kernel
    taps: list = field(default_factory=list)    # non-zero mask entries per kernel (0 for point)
    edges: list = field(default_factory=list)   # (ks, kd) unique, consumer-major order
    consumers: list = field(default_factory=list)
    producers: list = field(default_factory=list)


def kernel_costs(o: dict) -> tuple[int, int]:
    """nALU/nSFU of a kernel: explicit `cost`, else an opcode count (reading O1-d).
    Local: 2*nnz(mask)-1 multiply-adds plus the post program's ops."""
    if o.get("cost") is not None:
        return int(o["cost"][0]), int(o["cost"][1])
    prog = o["prog"] if o["kind"] == "point" else o["post"]
    n_sfu = sum(1 for t in prog if t[0] in SFU_OPS)
    n_alu = sum(1 for t in prog if t[0] not in NONARITH and t[0] not in SFU_OPS)
    if o["kind"] == "local":
        nnz = sum(1 for r in o["mask"] for v in r if v != 0.0)
        n_alu += 2 * max(nnz, 1) - 1
    return n_alu, n_sfu


def graph(spec: dict) -> Graph:
    ops = spec["ops"]
    n_in = spec["n_inputs"]
    g = Graph(n=len(ops), kind=[o["kind"] for o in ops], inputs=[list(o["inputs"]) for o in ops],
              n_inputs=n_in,
              rx=[len(o["mask"][0]) // 2 if o["kind"] == "local" else 0 for o in ops],
              ry=[len(o["mask"]) // 2 if o["kind"] == "local" else 0 for o in ops],
              mode=[o.get("mode") for o in ops], outputs=set(spec["outputs"]),
              bpp=4, cost=[kernel_costs(o) for o in ops], u8=spec["dtype"] == "u8x4",
              progs=[list(o["prog"] if o["kind"] == "point" else o["post"]) for o in ops],
              taps=[sum(1 for r in o["mask"] for v in r if v != 0.0) if o["kind"] == "local" else 0 for o in ops])
    g.consumers = [[] for _ in ops]
    g.producers = [[] for _ in ops]
    for kd, o in enumerate(ops):
        for img in o["inputs"]:
            if img >= n_in:
                ks = img - n_in
                if ks not in g.producers[kd]:
                    g.producers[kd].append(ks)
                    g.consumers[ks].append(kd)
                    g.edges.append((ks, kd))
    return g


# ------------------------------------------------------------- legality


def _dependence_legal(g: Graph, P: set) -> bool:
    """Reading O1-f of Fig. 2: one sink; every other kernel has all consumers inside
    and is not a pipeline output (Fig. 2c); every image a non-source kernel reads
    from outside P is also read by a source kernel (Fig. 2b legal / 2d illegal)."""
    sinks = [k for k in P if not any(c in P for c in g.consumers[k])]
    if len(sinks) != 1:
        return False
    for k in P:
        if k == sinks[0]:
            continue
        if (g.n_inputs + k) in g.outputs or any(c not in P for c in g.consumers[k]):
            return False
    sources = [k for k in P if not any(p in P for p in g.producers[k])]
    src_reads = {img for s in sources for img in g.inputs[s]}
    for k in P:
        if k in sources:
            continue
        for img in g.inputs[k]:
            inside = img >= g.n_inputs and (img - g.n_inputs) in P
            if not inside and img not in src_reads:
                return False
    return True


def f_mshared(g: Graph, k: int, m: Model) -> float:
    """Reading O1-h: staged-tile bytes of a local kernel, 0 for a point kernel."""
    if g.kind[k] != "local":
        return 0.0
    return float((m.tile_w + 2 * g.rx[k]) * (m.tile_h + 2 * g.ry[k]) * g.bpp)


def _resource_legal(g: Graph, P: set, m: Model) -> bool:
    """Eq. 2 with fMshared(vP) = sum over the block's local kernels."""
    loc = [k for k in sorted(P) if g.kind[k] == "local"]
    if not loc:
        return True
    s = 0.0
    for k in loc:
        s += f_mshared(g, k, m)
    mx = max(f_mshared(g, k, m) for k in loc)
    return s / mx <= m.c_mshared


def _header_legal(g: Graph, P: set) -> bool:
    """Same iteration space is enforced at pipeline creation;
    access-granularity reading (R-8): the local kernels of one fused block
    either all use REPEAT or none does."""
    loc = [k for k in P if g.kind[k] == "local"]
    rep = [g.mode[k] == "repeat" for k in loc]
    return all(rep) or not any(rep)


def context_legal(g: Graph, P: set, m: Model) -> bool:
    return _dependence_legal(g, P) and _resource_legal(g, P, m) and _header_legal(g, P)


# --------------------------------------------------------------- weights


@dataclass
class EdgeInfo:
    ks: int
    kd: int
    scenario: str     # "point", "p2l", "l2l"
    w: float          # benefit w + gamma (before clamping)
    ctx_legal: bool
    profitable: bool
    weight: tuple     # (q, eps)


def roofline_time(g: Graph, kernels: list, m: Model) -> float:
    """ROOFLINE reading R-20: SM-cycles per pixel of `kernels` (one kernel, or a
    producer followed by its consumer) fused into one kernel =
    max(M, C) + overlap * min(M, C).  M (DRAM): 4 B per distinct image read
    from outside plus the one output; C (issue): the kernels' issue slots per
    pixel (ISSUE_SLOTS per opcode, one per non-zero mask tap; x2 for u8x4's two
    SWAR channel pairs), the producer recomputed on the consumer's staged halo."""
    inside = {g.n_inputs + k for k in kernels}
    read = sorted({i for k in kernels for i in g.inputs[k] if i not in inside})
    per_ch = 2.0 if g.bpp == 4 and g.u8 else 1.0
    slots = []
    for pos, k in enumerate(kernels):
        c = float(sum(ISSUE_SLOTS.get(t[0], 1) for t in g.progs[k]) + g.taps[k]) * per_ch
        if pos == 0 and len(kernels) == 2 and g.kind[kernels[1]] == "local":
            kd = kernels[1]
            c *= (m.tile_w + 2 * g.rx[kd]) * (m.tile_h + 2 * g.ry[kd]) / (m.tile_w * m.tile_h)
        slots.append(c)
    dram = g.bpp * (len(read) + 1) / m.bw_bytes_clk
    issue = sum(slots) / m.issue_lanes_clk
    hi, lo = (dram, issue) if dram > issue else (issue, dram)
    return hi + m.overlap * lo


def benefit(g: Graph, ks: int, kd: int, m: Model) -> tuple[str, float]:
    """w for edge (ks, kd) by scenario, Eqs. 3-11, plus gamma (Eq. 12)."""
    if m.phi_mode == 2:                          # ROOFLINE reading R-20
        sc = "point" if g.kind[kd] == "point" else ("p2l" if g.kind[ks] == "point" else "l2l")
        w = roofline_time(g, [ks], m) + roofline_time(g, [kd], m) - roofline_time(g, [ks, kd], m)
        return sc, w + m.gamma
    IS = 1.0                                     # reading O1-c
    n_alu, n_sfu = g.cost[ks]
    costop = m.c_alu * n_alu + m.c_sfu * n_sfu   # Eq. 6
    is_ks = float(len(g.inputs[ks]))             # IS_ks: number of input images of ks
    if g.kind[kd] == "point":                    # point-based, Eq. 5 with Eq. 4
        return "point", IS * m.tg + m.gamma
    if m.phi_mode == 1:                          # STAGED reading (O1-g)
        fac = float((m.tile_w + 2 * g.rx[kd]) * (m.tile_h + 2 * g.ry[kd])) / float(m.tile_w * m.tile_h)
    elif g.kind[ks] == "point":
        fac = float((2 * g.rx[kd] + 1) * (2 * g.ry[kd] + 1))           # sz(kd), Eq. 7
    else:
        fac = float((2 * g.rx[kd] + 1 + 2 * g.rx[ks]) * (2 * g.ry[kd] + 1 + 2 * g.ry[ks]))  # Eq. 9 (O1-e)
    phi = costop * is_ks * fac                   # Eq. 7 / Eq. 10
    if g.kind[ks] == "point":
        return "p2l", IS * m.tg - phi + m.gamma  # Eq. 8
    delta_sh = IS * m.tg / m.ts if m.eq3_mode == 0 else IS * (m.tg - m.ts)   # Eq. 3 (O1-a)
    return "l2l", delta_sh - phi + m.gamma       # Eq. 11


def quantize(w: float) -> int:
    return int(math.floor(w * FIX + 0.5))


def edge_weights(g: Graph, m: Model) -> dict:
    """Alg. 1 lines 2-4: w_e = max(w + gamma, eps) (Eq. 12); illegal -> eps."""
    info = {}
    for ks, kd in g.edges:
        sc, w = benefit(g, ks, kd, m)
        prof = w > 0.0
        leg = context_legal(g, {ks, kd}, m)
        wt = (quantize(w), 0) if (prof and leg) else (0, 1)
        info[(ks, kd)] = EdgeInfo(ks, kd, sc, w, leg, prof, wt)
    return info


def is_legal(g: Graph, P: set, m: Model, info: dict) -> bool:
    """IsLegal(p) of Alg. 1 line 9; an unprofitable edge inside forbids the block (O1-g)."""
    if len(P) == 1:
        return True
    for (ks, kd), e in info.items():
        if ks in P and kd in P and not e.profitable:
            return False
    return context_legal(g, P, m)


# ---------------------------------------------------------- Stoer-Wagner


def _add(a, b):
    return (a[0] + b[0], a[1] + b[1])


def stoer_wagner(g: Graph, P: list, info: dict) -> tuple[list, list, tuple, int]:
    """Global minimum cut of the undirected view of block P (reading O1-j).
    Returns (t-side, rest, cut weight, number of phases)."""
    verts = sorted(P)
    idx = {v: i for i, v in enumerate(verts)}
    n = len(verts)
    W = [[(0, 0)] * n for _ in range(n)]
    for (ks, kd), e in info.items():
        if ks in idx and kd in idx:
            a, b = idx[ks], idx[kd]
            W[a][b] = _add(W[a][b], e.weight)
            W[b][a] = _add(W[b][a], e.weight)
    groups = [[v] for v in verts]
    active = list(range(n))          # positions in declaration order; merged vertex keeps s's slot
    best, best_group, phases = None, None, 0
    while len(active) > 1:
        phases += 1
        A = [active[0]]              # start vertex: first active vertex (dx in Fig. 3)
        conn = {v: W[active[0]][v] for v in active[1:]}
        last_conn = None
        while conn:
            # most tightly connected; ties -> lowest position (first encountered)
            v = min(conn, key=lambda u: (-conn[u][0], -conn[u][1], active.index(u)))
            last_conn = conn.pop(v)
            A.append(v)
            for u in conn:
                conn[u] = _add(conn[u], W[v][u])
        s, t = A[-2], A[-1]
        if best is None or last_conn < best:      # strict: keep the first one encountered
            best, best_group = last_conn, list(groups[t])
        # merge t into s
        groups[s] = groups[s] + groups[t]
        for u in range(n):
            W[s][u] = _add(W[s][u], W[t][u])
            W[u][s] = _add(W[u][s], W[u][t])
        W[s][s] = (0, 0)
        active.remove(t)
    side = sorted(best_group)
    rest = sorted(set(verts) - set(side))
    return side, rest, best, phases


# ---------------------------------------------------------------- Alg. 1


@dataclass
class Plan:
    blocks: list          # lists of kernel ids, topological (by sink)
    beta: tuple           # (q, eps)
    info: dict
    cuts: list            # [(block, side, cut weight, phases)] in processing order


def block_weight(P, info) -> tuple:
    s = (0, 0)
    for (ks, kd), e in info.items():
        if ks in P and kd in P:
            s = _add(s, e.weight)
    return s


def get_legal_partitions(spec: dict, m: Model = PAPER_PROFILE) -> Plan:
    """Alg. 1 GetLegalPartitions(G)."""
    g = graph(spec)
    info = edge_weights(g, m)                  # lines 2-4
    Sr = []                                    # line 5
    Sp = [list(range(g.n))]                    # line 6
    cuts = []
    while Sp:                                  # lines 7-17
        p = Sp.pop(0)
        if len(p) == 1 or is_legal(g, set(p), m, info):
            Sr.append(p)
        else:
            a, b, w, ph = stoer_wagner(g, p, info)
            cuts.append((p, a, w, ph))
            Sp += [a, b]
    Sr.sort(key=max)
    beta = (0, 0)
    for P in Sr:
        beta = _add(beta, block_weight(set(P), info))
    return Plan(Sr, beta, info, cuts)


# ------------------------------------------------------------ brute force


def _connected(g: Graph, P: list) -> bool:
    S = set(P)
    seen, stack = {P[0]}, [P[0]]
    while stack:
        v = stack.pop()
        for u in g.consumers[v] + g.producers[v]:
            if u in S and u not in seen:
                seen.add(u)
                stack.append(u)
    return len(seen) == len(S)


def brute_force(spec: dict, m: Model = PAPER_PROFILE) -> tuple[tuple, list]:
    """Maximum of Eq. 1 over all partitions into connected legal blocks
    (restricted-growth enumeration; Bell(n) partitions)."""
    g = graph(spec)
    info = edge_weights(g, m)
    n = g.n
    memo = {}

    def ok(block):
        key = frozenset(block)
        if key not in memo:
            memo[key] = (len(block) == 1 or (_connected(g, block) and is_legal(g, key, m, info)))
        return memo[key]

    best = [None, None]
    blocks: list[list[int]] = []

    # enumerate and check legality on completion
    def rec2(i):
        if i == n:
            if all(ok(b) for b in blocks):
                val = (0, 0)
                for b in blocks:
                    val = _add(val, block_weight(set(b), info))
                if best[0] is None or val > best[0]:
                    best[0], best[1] = val, sorted([sorted(b) for b in blocks], key=max)
            return
        for b in blocks:
            b.append(i)
            rec2(i + 1)
            b.pop()
        blocks.append([i])
        rec2(i + 1)
        blocks.pop()

    rec2(0)
    return best[0], best[1]


# ------------------------------------------------------ basic fusion [12]


def basic_legal(g: Graph, P: set, m: Model, info: dict) -> bool:
    """Reading R-18 of [12] as the paper describes it ("fusion
    ... only for point operator related fusion, namely point-to-point,
    local-to-point, and point-to-local"; Sobel's local-to-local
    and Unsharp's shared input "are rejected by the basic kernel fusion
    algorithm"): IsLegal, plus exactly one source kernel, no other kernel reads an
    image from outside P (a shared input counts as external), and no local kernel
    has a local kernel upstream inside P."""
    if len(P) == 1:
        return True
    if not is_legal(g, P, m, info):
        return False
    sources = [k for k in P if not any(p in P for p in g.producers[k])]
    if len(sources) != 1:
        return False
    for k in P:
        if k == sources[0]:
            continue
        for img in g.inputs[k]:
            if not (img >= g.n_inputs and (img - g.n_inputs) in P):
                return False
    for k in P:
        if g.kind[k] != "local":
            continue
        # every kernel upstream of k inside P
        up, stack = set(), [p for p in g.producers[k] if p in P]
        while stack:
            u = stack.pop()
            if u in up:
                continue
            up.add(u)
            stack += [p for p in g.producers[u] if p in P]
        if any(g.kind[u] == "local" for u in up):
            return False
    return True


def basic_fusion(spec: dict, m: Model = PAPER_PROFILE) -> list:
    """Pair-wise greedy fusion of [12] (reading R-18): visit the profitable edges by
    decreasing benefit w (ties: lower producer, then lower consumer); merge the two
    blocks the edge joins when their union is basic-legal; repeat full passes until
    nothing merges.  Returns the blocks sorted by their largest kernel."""
    g = graph(spec)
    info = edge_weights(g, m)
    block = {k: {k} for k in range(g.n)}          # kernel -> its block (shared sets)
    order = sorted((e for e in info.values() if e.profitable), key=lambda e: (-e.w, e.ks, e.kd))
    changed = True
    while changed:
        changed = False
        for e in order:
            a, b = block[e.ks], block[e.kd]
            if a is b:
                continue
            u = a | b
            if not basic_legal(g, u, m, info):
                continue
            for k in u:
                block[k] = u
            changed = True
    blocks = {id(b): sorted(b) for b in block.values()}
    return sorted(blocks.values(), key=max)


def min_cut_brute(g: Graph, P: list, info: dict) -> tuple:
    """Textbook check for Stoer-Wagner: min over all 2^(n-1)-1 bipartitions."""
    verts = sorted(P)
    n = len(verts)
    best = None
    for mask in range(1, 1 << (n - 1)):
        S = {verts[i] for i in range(n) if mask >> i & 1}
        w = (0, 0)
        for (ks, kd), e in info.items():
            if ks in P and kd in P and ((ks in S) != (kd in S)):
                w = _add(w, e.weight)
        if best is None or w < best:
            best = w
    return best

"""Pipeline descriptions as plain data (the workloads, not the method).

A pipeline is the paper's kernel DAG G = (V, E) (§II): a list
of kernels in declaration order, each a point or local operator
(§II-C-1) reading >= 1 same-size image and writing exactly 1.
Image ids are dense: inputs first (0 .. n_inputs-1), then kernel k writes image
n_inputs + k.  Both the oracle adapter (oracle/oracle.py) and the C-ABI binding
(paper_conf_cgo_qiaorht19_b200/kfuse.py) consume these dicts; this module holds
no arithmetic of the method (no stencil, no border map, no fusion, no weights).

Programs are postfix lists of (opcode-name, arg, imm); the op-IR is defined in
include/kfuse.h (kf_opcode).  Kernel bodies the paper does not print are the
readings of SURVEY.md §8(c) O2-f/g/h, restated in DESIGN.md §3.
"""
from __future__ import annotations

import math
import random
from typing import Any

# ---------------------------------------------------------------- op-IR sugar


def L(i: int):
    return ("LOAD", i, 0.0)


def C(v: float):
    return ("CONST", 0, float(v))


def op(name: str, arg: int = 0):
    return (name, arg, 0.0)


ADD, SUB, MUL, DIV = op("ADD"), op("SUB"), op("MUL"), op("DIV")
MIN, MAX, ABS, NEG = op("MIN"), op("MAX"), op("ABS"), op("NEG")
SQRT, EXP, LOG, POW = op("SQRT"), op("EXP"), op("LOG"), op("POW")
SAT, CLAMP, SELGT, LUT = op("SAT_U8"), op("CLAMP"), op("SELECT_GT"), op("LUT")


def SHR(n: int):
    return ("SHR", n, 0.0)


def SHL(n: int):
    return ("SHL", n, 0.0)


ACC = L(0)  # in a local op's post program, LOAD 0 is the accumulator

# ------------------------------------------------------------------ builder


class Pipeline:
    """Plain-data builder mirroring the C-ABI calls (kf_add_input / kf_add_*_op)."""

    def __init__(self, name: str, width: int, height: int, dtype: str):
        assert dtype in ("f32", "u8x4")
        self.d: dict[str, Any] = {"name": name, "width": int(width), "height": int(height),
                                  "dtype": dtype, "n_inputs": 0, "ops": [], "outputs": []}

    def _next_id(self) -> int:
        return self.d["n_inputs"] + len(self.d["ops"])

    def input(self) -> int:
        assert not self.d["ops"], "inputs must be declared before kernels"
        self.d["n_inputs"] += 1
        return self.d["n_inputs"] - 1

    def point(self, name: str, inputs: list[int], prog: list, cost=None, lut=None) -> int:
        out = self._next_id()
        self.d["ops"].append({"name": name, "kind": "point", "inputs": list(inputs), "prog": list(prog),
                              "cost": cost, "lut": None if lut is None else list(lut)})
        return out

    def local(self, name: str, inp: int, mask, mode: str, constant: float = 0.0, post=None, cost=None) -> int:
        out = self._next_id()
        m = [list(map(float, r)) for r in mask]
        assert len(m) % 2 == 1 and len(m[0]) % 2 == 1 and all(len(r) == len(m[0]) for r in m)
        self.d["ops"].append({"name": name, "kind": "local", "inputs": [inp], "mask": m, "mode": mode,
                              "constant": float(constant), "post": list(post or []), "cost": cost})
        return out

    def output(self, img: int) -> None:
        self.d["outputs"].append(img)

    def spec(self) -> dict:
        return self.d


def outer(col, row):
    return [[c * r for r in row] for c in col]


SOBEL_X = [[-1, 0, 1], [-2, 0, 2], [-1, 0, 1]]
SOBEL_Y = [[-1, -2, -1], [0, 0, 0], [1, 2, 1]]
GAUSS3 = [[1, 2, 1], [2, 4, 2], [1, 2, 1]]
GAUSS3_N = [[v / 16.0 for v in r] for r in GAUSS3]
BINOM5 = [1, 4, 6, 4, 1]
DERIV5 = [-1, -2, 0, 2, 1]

# ------------------------------------------------------------ paper workloads


def harris(width: int, height: int, mode: str = "clamp", k: float = 0.04, shitomasi: bool = False) -> dict:
    """Harris corner detector, Fig. 3 DAG: dx, dy local;
    sx, sy, sxy point; gx, gy, gxy local (Gaussian); hc point.  Bodies: SURVEY O2-f.
    nALU = 2 for the square/product kernels as in the worked example."""
    p = Pipeline("shitomasi" if shitomasi else "harris", width, height, "f32")
    i = p.input()
    dx = p.local("dx", i, SOBEL_X, mode)
    dy = p.local("dy", i, SOBEL_Y, mode)
    sx = p.point("sx", [dx], [L(0), L(0), MUL], cost=(2, 0))
    sy = p.point("sy", [dy], [L(0), L(0), MUL], cost=(2, 0))
    sxy = p.point("sxy", [dx, dy], [L(0), L(1), MUL], cost=(2, 0))
    gx = p.local("gx", sx, GAUSS3_N, mode)
    gy = p.local("gy", sy, GAUSS3_N, mode)
    gxy = p.local("gxy", sxy, GAUSS3_N, mode)
    if shitomasi:
        # lambda_min = 1/2 ((gx+gy) - sqrt((gx-gy)^2 + 4 gxy^2))   (O2-f)
        prog = [L(0), L(1), ADD, L(0), L(1), SUB, L(0), L(1), SUB, MUL, C(4.0), L(2), MUL, L(2), MUL, ADD,
                SQRT, SUB, C(0.5), MUL]
        hc = p.point("st", [gx, gy, gxy], prog)
    else:
        # R = gx*gy - gxy^2 - k (gx+gy)^2
        prog = [L(0), L(1), MUL, L(2), L(2), MUL, SUB, C(k), L(0), L(1), ADD, MUL, L(0), L(1), ADD, MUL, SUB]
        hc = p.point("hc", [gx, gy, gxy], prog)
    p.output(hc)
    return p.spec()


def unsharp(width: int, height: int, mode: str = "clamp") -> dict:
    """Unsharp: one local blur then three point kernels, all reading the input
    (Fig. 2b shape).  Bodies: SURVEY O2-g."""
    p = Pipeline("unsharp", width, height, "f32")
    i = p.input()
    blur = p.local("blur", i, GAUSS3_N, mode)
    p1 = p.point("p1", [i, blur], [L(0), L(1), SUB])
    p2 = p.point("p2", [i, p1], [L(0), C(1.5), L(1), MUL, ADD])
    p3 = p.point("p3", [i, p2], [L(0), L(1), L(0), SUB, C(-0.125), C(0.125), CLAMP, ADD])
    p.output(p3)
    return p.spec()


def sobel(width: int, height: int, mode: str = "clamp") -> dict:
    """Sobel: two local gradients then the magnitude."""
    p = Pipeline("sobel", width, height, "f32")
    i = p.input()
    dx = p.local("dx", i, SOBEL_X, mode)
    dy = p.local("dy", i, SOBEL_Y, mode)
    mag = p.point("mag", [dx, dy], [L(0), L(0), MUL, L(1), L(1), MUL, ADD, SQRT])
    p.output(mag)
    return p.spec()


def enhance(width: int, height: int, mode: str = "mirror", gamma1: float = 0.8, gamma2: float = 1.2) -> dict:
    """Enhancement: geometric-mean filter then gamma point ops, a chain.
    Geometric mean as exp(mean(log(x + 1/256)))."""
    p = Pipeline("enhance", width, height, "f32")
    i = p.input()
    lg = p.point("log", [i], [L(0), C(1.0 / 256.0), ADD, LOG])
    box = p.local("box", lg, [[1.0 / 9.0] * 3] * 3, mode)
    gm = p.point("gmean", [box], [L(0), EXP])
    g1 = p.point("gamma1", [gm], [L(0), C(gamma1), POW])
    g2 = p.point("gamma2", [g1], [L(0), C(gamma2), POW, C(1.0), MIN])
    p.output(g2)
    return p.spec()


def gamma_lut(g: float = 0.8) -> list[int]:
    return [min(255, int(math.floor(255.0 * (v / 255.0) ** g + 0.5))) for v in range(256)]


def deep10(width: int, height: int, mode: str = "mirror") -> dict:
    """C4: synthetic 10-kernel uint8 RGBA pipeline, 4 local 5x5 + 6 point.
    Integer semantics per channel, int32 accumulators, >> arithmetic, sat = clamp [0,255]."""
    p = Pipeline("deep10", width, height, "u8x4")
    i = p.input()
    bb = outer(BINOM5, BINOM5)
    k0 = p.local("k0", i, bb, mode, post=[ACC, C(128), ADD, SHR(8), SAT])
    k1 = p.point("k1", [i, k0], [L(0), L(1), SUB, C(128), ADD, SAT])
    k2 = p.local("k2", k1, outer(BINOM5, DERIV5), mode, post=[ACC, SHR(5), C(128), ADD, SAT])
    k3 = p.local("k3", k1, outer(DERIV5, BINOM5), mode, post=[ACC, SHR(5), C(128), ADD, SAT])
    k4 = p.point("k4", [k2, k3], [L(0), L(1), ADD, C(1), ADD, SHR(1)])
    k5 = p.local("k5", k4, bb, mode, post=[ACC, C(128), ADD, SHR(8), SAT])
    k6 = p.point("k6", [k5], [L(0), LUT], lut=gamma_lut(0.8))
    k7 = p.point("k7", [i, k6], [C(3), L(0), MUL, L(1), ADD, C(2), ADD, SHR(2)])
    k8 = p.point("k8", [k7, k0], [L(0), L(0), L(1), SUB, C(3), MUL, SHR(1), ADD, SAT])
    k9 = p.point("k9", [k8, i], [L(0), L(1), ADD, C(1), ADD, SHR(1)])
    p.output(k9)
    return p.spec()


def copy(width: int, height: int, mode: str = "clamp") -> dict:
    """Diagnostic: one point kernel out = in (the streaming path's memory-side ceiling)."""
    p = Pipeline("copy", width, height, "f32")
    i = p.input()
    p.output(p.point("copy", [i], [L(0)]))
    return p.spec()


def blur(width: int, height: int, mode: str = "clamp") -> dict:
    """Diagnostic: one 3x3 Gaussian local kernel."""
    p = Pipeline("blur", width, height, "f32")
    i = p.input()
    p.output(p.local("blur", i, GAUSS3_N, mode))
    return p.spec()


def swar_stress(W, H, mode="mirror"):
    """u8x4 kernels on both sides of the SWAR interval check: linear forms with
    negative ranges, MIN/MAX of differently biased values, NEG/SHL, clamps, a short
    LUT with entries above 255, a CONSTANT border at 255 -- and kernels that must
    fall back to int32 (a 16-bit-overflowing mask, ABS, DIV, SELECT, a variable
    product)."""
    ACC = L(0)
    p = Pipeline("swar_stress", W, H, "u8x4")
    i = p.input()
    a = p.local("a", i, [[1, -2, 1], [-2, 4, -2], [1, -2, 1]], "constant", constant=255.0,
                post=[ACC, C(64), ADD, SHR(2), SAT])
    b = p.point("b", [i, a], [L(0), L(1), SUB, NEG, L(0), MAX, C(1), op("SHL", 2), ADD, SHR(3), SAT])
    c = p.point("c", [a, b], [L(0), C(3), MUL, L(1), MIN, C(10), C(200), CLAMP])
    d = p.point("d", [c], [L(0), LUT], lut=[(7 * v) % 301 for v in range(100)])
    big = [[60] * 5 for _ in range(5)]
    e = p.local("e", d, big, mode, post=[ACC, SHR(12), SAT])                 # 16-bit overflow: int32
    f = p.point("f", [e, b], [L(0), L(1), SUB, ABS, C(255), MIN])           # ABS: int32
    g = p.point("g", [f, c], [L(0), C(7), MUL, L(1), C(1), ADD, DIV, SAT])  # DIV: int32
    h = p.point("h", [g, a, b, d], [L(0), L(1), L(2), L(3), SELGT])          # SELECT: int32
    k = p.point("k", [h, g], [L(0), L(1), MUL, SHR(8), SAT])                 # variable product: int32
    m = p.local("m", k, [[1, 2, 1], [2, 4, 2], [1, 2, 1]], "constant", constant=255.0,
                post=[ACC, C(8), ADD, SHR(4), SAT])
    p.output(m)
    return p.spec()


def two_input(width: int, height: int, mode: str = "clamp") -> dict:
    """Test workload with two input images (multi-input row bands / peer halos):
    a 5x5 binomial blur of input 0, a Sobel-x of input 1, combined pointwise with
    input 0 (a shared external input, Fig. 2b shape)."""
    p = Pipeline("two_input", width, height, "f32")
    a, b = p.input(), p.input()
    bl = p.local("blur", a, [[v / 256.0 for v in r] for r in outer(BINOM5, BINOM5)], mode)
    dx = p.local("dx", b, SOBEL_X, mode)
    p.output(p.point("mix", [bl, dx, a], [L(0), L(1), MUL, L(2), ADD]))
    return p.spec()


def fig4(mode: str = "clamp") -> dict:
    """Fig. 4: two unnormalised 3x3 Gaussian local kernels on a 5x5 image."""
    p = Pipeline("fig4", 5, 5, "f32")
    i = p.input()
    a = p.local("kp", i, GAUSS3, mode)
    b = p.local("kc", a, GAUSS3, mode)
    p.output(b)
    return p.spec()


FIG4_IMAGE = [[1, 3, 7, 7, 6], [3, 7, 9, 6, 8], [5, 4, 3, 2, 1], [4, 1, 2, 1, 2], [5, 2, 2, 4, 2]]

# ------------------------------------------------------- random DAGs (tests)

MODES = ["clamp", "mirror", "mirror101", "repeat", "constant"]


def random_pipeline(rng: random.Random, width: int, height: int, dtype: str, n_kernels: int,
                    modes=None, max_radius: int = 2, asym: float = 0.0) -> dict:
    """Random connected DAG of point/local kernels for property tests.  Values stay
    bounded: f32 programs are convex-ish combinations, u8x4 programs saturate.
    max_radius bounds each mask's radius per axis; with probability `asym` a local
    kernel takes a strongly asymmetric shape instead (1x7, 9x1, 1x9, 7x1, 3x7, 9x5
    masks as (rows x cols)).  asym = 0 draws no extra random numbers, so the
    default stream of DAGs is unchanged."""
    modes = modes or MODES
    p = Pipeline(f"rand_{dtype}_{n_kernels}", width, height, dtype)
    n_in = rng.choice([1, 1, 2])
    imgs = [p.input() for _ in range(n_in)]
    for k in range(n_kernels):
        # prefer the most recent images so the DAG is deep and connected
        def pick():
            w = [1.0 + 3.0 * (j >= len(imgs) - 2) for j in range(len(imgs))]
            return rng.choices(imgs, weights=w)[0]
        if rng.random() < 0.5:
            r = rng.randint(1, max_radius)
            ry = rng.choice([r, rng.randint(0, max_radius)])
            rx = rng.choice([r, rng.randint(0, max_radius)])
            if rx == 0 and ry == 0:
                rx = 1
            if asym and rng.random() < asym:
                ry, rx = rng.choice([(0, 3), (4, 0), (0, 4), (3, 0), (1, 3), (4, 2)])
            mode = rng.choice(modes)
            src = pick()
            if dtype == "f32":
                if rng.random() < 0.5:
                    col = [rng.choice([1, 2, 3, -1]) for _ in range(2 * ry + 1)]
                    row = [rng.choice([1, 2, -2, 1]) for _ in range(2 * rx + 1)]
                    mask = outer(col, row)
                else:
                    mask = [[rng.randint(-3, 4) for _ in range(2 * rx + 1)] for _ in range(2 * ry + 1)]
                s = sum(abs(v) for r_ in mask for v in r_) or 1
                mask = [[v / s for v in r_] for r_ in mask]
                post = rng.choice([[], [ACC, C(0.5), ADD], [ACC, ABS]])
                const = rng.choice([0.0, 0.25, 1.0])
            else:
                col = [rng.randint(0, 4) for _ in range(2 * ry + 1)]
                row = [rng.randint(-2, 4) for _ in range(2 * rx + 1)]
                if sum(col) == 0:
                    col[ry] = 1
                mask = outer(col, row) if rng.random() < 0.6 else \
                    [[rng.randint(-2, 5) for _ in range(2 * rx + 1)] for _ in range(2 * ry + 1)]
                s = sum(abs(v) for r_ in mask for v in r_) or 1
                sh = max(0, int(math.ceil(math.log2(s))))
                post = [ACC, C(1 << max(sh - 1, 0)), ADD, SHR(sh), C(rng.choice([0, 64, 128])), ADD, SAT]
                const = float(rng.choice([0, 17, 255]))
            imgs.append(p.local(f"l{k}", src, mask, mode, constant=const, post=post))
        else:
            n = rng.choice([1, 2, 2, 3])
            ins = []
            for _ in range(n):
                c = pick()
                if c not in ins:
                    ins.append(c)
            if dtype == "f32":
                prog = [L(0)]
                for j in range(1, len(ins)):
                    prog += [L(j), rng.choice([ADD, SUB, MAX, MIN])]
                prog += rng.choice([[C(0.5), MUL], [L(0), MUL, C(0.25), MUL], [ABS], [C(0.1), ADD]])
            else:
                prog = [L(0)]
                for j in range(1, len(ins)):
                    prog += [L(j), rng.choice([ADD, SUB, MAX, MIN])]
                prog += rng.choice([[C(1), ADD, SHR(1)], [C(128), ADD, SAT], [SAT], [C(3), MUL, SHR(2), SAT]])
                if len(ins) == 1 and rng.random() < 0.3:
                    prog = [L(0), LUT]
            lut = None
            if any(t[0] == "LUT" for t in prog):
                lut = [rng.randint(0, 255) for _ in range(256)]
            imgs.append(p.point(f"p{k}", ins, prog, lut=lut))
    # every kernel nobody consumes is an output; sometimes an inner one is too
    used = {i for o in p.d["ops"] for i in o["inputs"]}
    for img in imgs[n_in:]:
        if img not in used:
            p.output(img)
    inner = [img for img in imgs[n_in:] if img in used]
    if inner and rng.random() < 0.3:
        p.output(rng.choice(inner))
    return p.spec()


WORKLOADS = {
    "harris": harris,
    "shitomasi": lambda w, h, mode="clamp": harris(w, h, mode, shitomasi=True),
    "unsharp": unsharp,
    "sobel": sobel,
    "enhance": enhance,
    "deep10": deep10,
    "copy": copy,
    "blur": blur,
    "two_input": two_input,
}

# BASELINE.json configs: (workload, W, H, seed)
CONFIGS = {
    "C1": ("harris", 256, 256, 1),
    "C2": ("unsharp", 2048, 2048, 2),
    "C3": ("harris", 4096, 4096, 3),
    "C3s": ("shitomasi", 4096, 4096, 3),
    "C4": ("deep10", 7680, 4320, 4),
    "C5": ("harris", 16384, 16384, 5),
}


def config(name: str) -> tuple[dict, int]:
    wl, w, h, seed = CONFIGS[name]
    return WORKLOADS[wl](w, h), seed

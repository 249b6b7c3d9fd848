"""Pins for the oracle's op-IR interpreter (oracle/kf_oracle.c run_f / run_i),
opcode by opcode, against numpy on the same values.

The op-IR semantics are the interface's (include/kfuse.h, kf_opcode): postfix
stack machine, "pop b, pop a, push a op b", CLAMP pops hi then lo then x,
SELECT_GT pops d, c, b, a and pushes (a > b) ? c : d, int DIV truncates with
x/0 = 0, SHR is an arithmetic (floor) shift, LUT clamps its index, and a U8X4
kernel's result is saturated to [0,255] when stored.  Point bodies are the
paper's point operators out(y,x) = f(in_1(y,x), ..., in_n(y,x))
(§II-C-1); the workload bodies that use these opcodes
(Enhance: LOG/EXP/POW/MIN, Unsharp: CLAMP, deep10: SHR/LUT/SAT, swar_stress:
the rest) are DESIGN.md R-15.

Every program is built so that a plausible slip -- swapped operands of POW,
SUB or DIV, CLAMP's lo/hi popped in the wrong order, SELECT_GT's c/d swapped,
DIV rounding toward -inf instead of 0, SHR truncating instead of flooring, a
LUT index wrapping instead of clamping, SAT skipped in favour of the store
saturation -- changes the result on many pixels.  Expected values come from
numpy written directly from the definitions above, never from the oracle.
CPU only.
"""
import zlib

import numpy as np
import pytest

from kf_inputs import pipelines as P
from oracle import oracle as O

W, H = 16, 12
L, C, op = P.L, P.C, P.op
ADD, SUB, MUL = P.ADD, P.SUB, P.MUL


def _point_spec(dtype, n_in, prog, lut=None):
    p = P.Pipeline("opcode", W, H, dtype)
    ins = [p.input() for _ in range(n_in)]
    p.output(p.point("k", ins, prog, lut=lut))
    return p.spec()


def _f32_inputs(seed, n):
    rng = np.random.default_rng(seed)
    # distinct, positive, well away from 0 and 1 so that operand order matters everywhere
    return [(0.05 + 1.9 * rng.random((H, W))).astype(np.float32) for _ in range(n)]


def _u8_inputs(seed, n):
    rng = np.random.default_rng(seed)
    return [rng.integers(0, 256, (H, W, 4), dtype=np.uint8) for _ in range(n)]


def _run(spec, ins):
    return O.run(spec, ins)[spec["outputs"][0]]


# ------------------------------------------------------------------ f32 (fp64 in the oracle)

def _f(ins):
    return [a.astype(np.float64) for a in ins]


F32_CASES = {
    # name: (n_inputs, program, numpy definition on fp64 copies of the inputs)
    "CONST": (1, [L(0), C(0.3), ADD], lambda a: a[0] + 0.3),
    "ADD": (2, [L(0), L(1), ADD], lambda a: a[0] + a[1]),
    "SUB": (2, [L(0), L(1), SUB], lambda a: a[0] - a[1]),
    "MUL": (2, [L(0), L(1), op("MUL")], lambda a: a[0] * a[1]),
    "DIV": (2, [L(0), L(1), op("DIV")], lambda a: a[0] / a[1]),
    "MIN": (2, [L(0), L(1), op("MIN")], lambda a: np.minimum(a[0], a[1])),
    "MAX": (2, [L(0), L(1), op("MAX")], lambda a: np.maximum(a[0], a[1])),
    "ABS": (1, [L(0), C(1.0), SUB, op("ABS")], lambda a: np.abs(a[0] - 1.0)),
    "NEG": (2, [L(0), op("NEG"), L(1), ADD], lambda a: a[1] - a[0]),
    "SQRT": (1, [L(0), op("SQRT")], lambda a: np.sqrt(a[0])),
    "EXP": (1, [L(0), op("EXP")], lambda a: np.exp(a[0])),
    "LOG": (1, [L(0), op("LOG")], lambda a: np.log(a[0])),
    "POW": (2, [L(0), L(1), op("POW")], lambda a: np.power(a[0], a[1])),
    "POW_CONST": (1, [L(0), C(0.8), op("POW")], lambda a: np.power(a[0], 0.8)),
    "CLAMP": (1, [L(0), C(0.6), C(1.3), op("CLAMP")], lambda a: np.clip(a[0], 0.6, 1.3)),
    "CLAMP_LOADED": (3, [L(0), L(1), C(0.5), MUL, L(2), C(1.0), ADD, op("CLAMP")],
                     lambda a: np.minimum(np.maximum(a[0], 0.5 * a[1]), a[2] + 1.0)),
    "SELECT_GT": (4, [L(0), L(1), L(2), L(3), op("SELECT_GT")],
                  lambda a: np.where(a[0] > a[1], a[2], a[3])),
    # Unsharp's p3 body (R-15): in + clamp(p2 - in, -0.125, 0.125)
    "UNSHARP_P3": (2, [L(0), L(1), L(0), SUB, C(-0.125), C(0.125), op("CLAMP"), ADD],
                   lambda a: a[0] + np.clip(a[1] - a[0], -0.125, 0.125)),
    # Enhance's chain (R-15): min(pow(exp(log(x + 1/256)), 1.2), 1)
    "ENHANCE_CHAIN": (1, [L(0), C(1 / 256), ADD, op("LOG"), op("EXP"), C(1.2), op("POW"), C(1.0), op("MIN")],
                      lambda a: np.minimum(np.power(np.exp(np.log(a[0] + 1 / 256)), 1.2), 1.0)),
}

# libm and numpy may differ by an ulp on transcendental functions; arithmetic is exact
_TRANSCENDENTAL = {"EXP", "LOG", "POW", "POW_CONST", "ENHANCE_CHAIN"}


@pytest.mark.parametrize("name", sorted(F32_CASES))
def test_f32_opcode(name):
    n, prog, ref = F32_CASES[name]
    ins = _f32_inputs(zlib.crc32(name.encode()) % 1000, n)
    got = _run(_point_spec("f32", n, prog), ins)
    want = ref(_f(ins))
    if name in _TRANSCENDENTAL:
        np.testing.assert_allclose(got, want, rtol=4e-16, atol=0)
    else:
        np.testing.assert_array_equal(got, want)


def test_f32_select_gt_ties_take_d():
    """a > b is strict: equal operands select d."""
    a = _f32_inputs(5, 1)[0]
    spec = _point_spec("f32", 1, [L(0), L(0), C(1.0), C(2.0), op("SELECT_GT")])
    assert np.all(_run(spec, [a]) == 2.0)


def test_f32_local_post_program_reads_acc():
    """In a local op's post program LOAD 0 is the accumulator (kfuse.h)."""
    p = P.Pipeline("post", W, H, "f32")
    i = p.input()
    p.output(p.local("l", i, [[0, 0, 0], [0, 2, 0], [0, 0, 0]], "clamp", post=[L(0), C(3.0), op("SUB"), C(0.5),
                                                                                 op("POW")]))
    a = _f32_inputs(6, 1)[0]
    a = a + np.float32(2.0)
    got = _run(p.spec(), [a])
    np.testing.assert_allclose(got, np.power(2.0 * a.astype(np.float64) - 3.0, 0.5), rtol=4e-16)


# ------------------------------------------------------------ u8x4 (exact int, saturated store)

def _i(ins):
    return [a.astype(np.int64) for a in ins]


def _trunc_div(a, b):
    q = np.abs(a) // np.where(b == 0, 1, np.abs(b))
    q = np.where(np.sign(a) * np.sign(b) < 0, -q, q)
    return np.where(b == 0, 0, q)


def _sat(v):
    return np.clip(v, 0, 255)


LUT100 = [(37 * v + 11) % 400 for v in range(100)]   # entries above 255 too: the store saturates

INT_CASES = {
    "CONST_TRUNC": (1, [L(0), C(2.7), ADD, C(-2.7), ADD], lambda a: a[0]),            # 2 and -2
    "ADD": (2, [L(0), L(1), ADD, op("SHR", 1)], lambda a: (a[0] + a[1]) >> 1),
    "SUB": (2, [L(0), L(1), op("SUB"), C(255), ADD, P.SHR(1)], lambda a: (a[0] - a[1] + 255) >> 1),
    "MUL": (2, [L(0), L(1), op("MUL"), P.SHR(8)], lambda a: (a[0] * a[1]) >> 8),
    "DIV": (2, [L(0), C(300), op("SUB"), L(1), C(1), ADD, op("DIV"), C(128), ADD],
            lambda a: _sat(_trunc_div(a[0] - 300, a[1] + 1) + 128)),
    "DIV_BY_ZERO": (2, [L(0), L(1), C(0), op("MUL"), op("DIV"), C(7), ADD], lambda a: a[0] * 0 + 7),
    "DIV_OPERANDS": (2, [C(4000), L(0), C(1), ADD, op("DIV")], lambda a: _sat(4000 // (a[0] + 1))),
    "MIN": (2, [L(0), L(1), op("MIN")], lambda a: np.minimum(a[0], a[1])),
    "MAX": (2, [L(0), L(1), op("MAX")], lambda a: np.maximum(a[0], a[1])),
    "ABS": (1, [L(0), C(128), op("SUB"), op("ABS"), P.SHL(1)], lambda a: _sat(np.abs(a[0] - 128) * 2)),
    "NEG": (2, [L(0), op("NEG"), L(1), ADD, C(255), ADD, P.SHR(1)], lambda a: (a[1] - a[0] + 255) >> 1),
    "SHR_FLOOR": (1, [L(0), C(200), op("SUB"), P.SHR(3), C(128), ADD], lambda a: ((a[0] - 200) >> 3) + 128),
    "SHL": (1, [L(0), C(60), op("SUB"), P.SHL(2), C(128), ADD], lambda a: _sat(((a[0] - 60) << 2) + 128)),
    "SAT_U8": (1, [L(0), C(3), op("MUL"), C(200), op("SUB"), op("SAT_U8"), P.SHR(1)],
               lambda a: _sat(3 * a[0] - 200) >> 1),
    "CLAMP": (1, [L(0), C(50), C(180), op("CLAMP")], lambda a: np.clip(a[0], 50, 180)),
    "CLAMP_LOADED": (3, [L(0), L(1), P.SHR(1), L(2), P.SHR(1), C(128), ADD, op("CLAMP")],
                     lambda a: np.minimum(np.maximum(a[0], a[1] >> 1), (a[2] >> 1) + 128)),
    "SELECT_GT": (4, [L(0), L(1), L(2), L(3), op("SELECT_GT")], lambda a: np.where(a[0] > a[1], a[2], a[3])),
    "LUT_CLAMPED_INDEX": (1, [L(0), C(100), op("SUB"), op("LUT")],
                          lambda a: _sat(np.array(LUT100)[np.clip(a[0] - 100, 0, 99)])),
}


@pytest.mark.parametrize("name", sorted(INT_CASES))
def test_int_opcode(name):
    n, prog, ref = INT_CASES[name]
    ins = _u8_inputs(1 + zlib.crc32(name.encode()) % 1000, n)
    lut = LUT100 if "LUT" in name else None
    got = _run(_point_spec("u8x4", n, prog, lut=lut), ins)
    want = _sat(ref(_i(ins))).astype(np.uint8)
    np.testing.assert_array_equal(got, want)


def test_int_store_saturates():
    """A U8X4 kernel's result is saturated to [0,255] when stored (kfuse.h)."""
    a = _u8_inputs(9, 1)[0]
    got = _run(_point_spec("u8x4", 1, [L(0), C(2), op("MUL"), C(100), op("SUB")]), [a])
    np.testing.assert_array_equal(got, _sat(2 * a.astype(np.int64) - 100).astype(np.uint8))


def test_int_channels_independent():
    """u8x4 programs run per channel (R-16): a channel-permuted input permutes the output."""
    a, b = _u8_inputs(10, 2)
    spec = _point_spec("u8x4", 2, [L(0), L(1), op("SUB"), C(255), ADD, P.SHR(1)])
    got = _run(spec, [a, b])
    perm = [2, 0, 3, 1]
    got_p = _run(spec, [np.ascontiguousarray(a[..., perm]), np.ascontiguousarray(b[..., perm])])
    np.testing.assert_array_equal(got_p, got[..., perm])


def test_int_overflow_is_reported():
    """int32 accumulator overflow is an error, not a silent wrap (kf_oracle.c chk)."""
    a = np.full((H, W, 4), 255, np.uint8)
    spec = _point_spec("u8x4", 1, [L(0), C(1 << 20), op("MUL"), C(1 << 20), op("MUL"), op("SAT_U8")])
    with pytest.raises(RuntimeError):
        _run(spec, [a])

"""Pins for the image oracle (oracle/kf_oracle.c) against what the paper and the
mathematics fix -- never against the oracle itself or the CUDA path.

Each test names the passage it pins.  CPU only."""
import json
import os
import random

import numpy as np
import pytest
import scipy.ndimage as ndi

from kf_inputs import gen
from kf_inputs import pipelines as P
from oracle import oracle as O

MODES = ["clamp", "mirror", "mirror101", "repeat", "constant"]
NP_PAD = {"clamp": "edge", "mirror": "symmetric", "mirror101": "reflect", "repeat": "wrap"}


# ------------------------------------------------------------- Fig. 4 pins

@pytest.fixture(scope="module")
def fig4(golden_dir):
    with open(os.path.join(golden_dir, "fig4.json")) as f:
        return json.load(f)


def test_fig4a_body_fusion_interior(fig4):
    """Fig. 4a: interior intermediate and output 992."""
    s = P.fig4("clamp")
    r = O.run(s, [np.array(fig4["image_5x5"], np.float32)], [1, 2])
    assert r[1][1:4, 1:4].tolist() == fig4["fig4a_intermediate_interior"]
    assert r[2][2, 2] == fig4["fig4a_output_center"]


def test_fig4c_correct_border_fusion(fig4):
    """Fig. 4c: clamp+conv+clamp+conv -> 763 at (0,0); the
    clamped intermediate window equals the figure's."""
    s = P.fig4("clamp")
    r = O.run(s, [np.array(fig4["image_5x5"], np.float32)], [1, 2])
    inter = r[1]
    win = [[inter[max(y, 0), max(x, 0)] for x in (-1, 0, 1)] for y in (-1, 0, 1)]
    assert win == fig4["fig4c_intermediate_window_topleft"]
    assert r[2][0, 0] == fig4["fig4c_output_topleft"]
    img = np.array(fig4["image_5x5"])
    ex = [[img[max(y, 0), max(x, 0)] for x in range(-1, 3)] for y in range(-1, 3)]
    assert ex == fig4["fig4c_exchanged_input_window"]


def test_fig4b_pad_once_is_a_negative_control(fig4):
    """Fig. 4b: padding once and convolving twice is WRONG at
    the border; the paper's own intermediate gives 684 (it prints 648)."""
    img = np.array(fig4["image_5x5"], np.float64)
    m = np.array(fig4["mask"], np.float64)
    pad = np.pad(img, 2, mode="edge")
    a = ndi.correlate(pad, m, mode="constant")[1:-1, 1:-1]      # 7x7 intermediate of padded
    win = a[0:3, 0:3]
    assert win.tolist() == fig4["fig4b_intermediate_window_topleft"]
    naive = float((win * m).sum())
    assert naive == fig4["fig4b_output_topleft_recomputed"]
    r = O.run(P.fig4("clamp"), [img.astype(np.float32)], [2])[2]
    assert r[0, 0] != naive and r[0, 0] == 763


# ------------------------------------------------------- border accessor

@pytest.mark.parametrize("mode", ["clamp", "mirror", "mirror101", "repeat"])
@pytest.mark.parametrize("n", [1, 2, 3, 5, 8])
def test_border_map_matches_numpy_pad(mode, n):
    """border modes equal numpy.pad's edge/symmetric/reflect/wrap,
    including repeated folding when the halo exceeds the image."""
    if mode == "mirror101" and n == 1:
        pytest.skip("numpy reflect of a length-1 axis is the identity; covered below")
    h = 3 * n + 2
    ref = np.pad(np.arange(n), h, mode=NP_PAD[mode])
    got = [O.border(p, n, mode) for p in range(-h, n + h)]
    assert got == ref.tolist()


def test_border_constant_and_degenerate():
    assert O.border(-1, 5, "constant") == -1 and O.border(5, 5, "constant") == -1
    assert O.border(2, 5, "constant") == 2
    assert O.border(-3, 1, "mirror101") == 0


# ------------------------------------------------- 8x8 hand values (A5)

def _single_local(w, h, mask, mode, constant=0.0, dtype="f32"):
    p = P.Pipeline("one", w, h, dtype)
    i = p.input()
    o = p.local("l", i, mask, mode, constant=constant)
    p.output(o)
    return p.spec()


@pytest.mark.parametrize("name", ["gauss3", "sobel_x", "binom5"])
@pytest.mark.parametrize("mode", MODES)
def test_ramp8_hand_values(golden_dir, name, mode):
    """North star: hand-computed mask results with clamp/mirror/constant borders on
    8x8 images (tests/golden/ramp8.json)."""
    with open(os.path.join(golden_dir, "ramp8.json")) as f:
        g = json.load(f)
    e = g[name]
    mask = e["mask"] if "mask" in e else P.outer(e["mask_outer"], e["mask_outer"])
    img = (8 * np.arange(8)[:, None] + np.arange(8)[None, :]).astype(np.float32)
    r = O.run(_single_local(8, 8, mask, mode), [img])
    out = list(r.values())[0]
    assert [out[y, x] for y, x in g["points"]] == e[mode]


# ------------------------------------------- library cross-check (scipy)

SCIPY_MODE = {"clamp": "nearest", "mirror": "reflect", "mirror101": "mirror", "repeat": "wrap",
              "constant": "constant"}


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("shape", [(9, 7), (3, 11), (16, 16)])
def test_local_op_equals_scipy_correlate(mode, shape):
    """A single local operator is textbook correlation with a border mode
    (scipy.ndimage.correlate).  Non-square, non-symmetric masks
    catch transposed or flipped operands."""
    rng = np.random.default_rng(7)
    H, W = shape
    img = rng.integers(0, 50, size=(H, W)).astype(np.float32)
    for mh, mw in [(3, 3), (5, 3), (1, 5), (5, 5)]:
        mask = rng.integers(-3, 4, size=(mh, mw)).astype(np.float64)
        if mode in ("mirror", "mirror101") and (mh // 2 >= H or mw // 2 >= W):
            continue      # scipy folds differently once the halo exceeds the axis
        c = 2.5
        ref = ndi.correlate(img.astype(np.float64), mask, mode=SCIPY_MODE[mode], cval=c)
        got = list(O.run(_single_local(W, H, mask.tolist(), mode, c), [img]).values())[0]
        np.testing.assert_array_equal(got, ref)


def test_u8x4_local_channels_independent():
    """u8x4: each channel is its own image (interleaved RGBA), integer correlation."""
    rng = np.random.default_rng(3)
    img = rng.integers(0, 256, size=(6, 9, 4)).astype(np.uint8)
    mask = [[1, 2, 1], [0, 3, 0], [1, 0, 2]]
    s = _single_local(9, 6, mask, "mirror", dtype="u8x4")
    s["ops"][0]["post"] = [P.ACC, P.SHR(4), P.SAT]
    got = O.run(s, [img])[1]
    for ch in range(4):
        ref = ndi.correlate(img[..., ch].astype(np.int64), np.array(mask), mode="reflect")
        ref = np.clip(np.floor_divide(ref, 16), 0, 255)
        np.testing.assert_array_equal(got[..., ch], ref)


# ------------------------------------------------ closed forms (Harris)

def test_harris_ramp_closed_form():
    """I = a x + b y: interior dx = 8a, dy = 8b (Sobel gains 4 x 2), Gaussian sums to 1,
    so gx = 64a^2, gy = 64b^2, gxy = 64ab, det = 0 and R = -k (64 (a^2+b^2))^2;
    Shi-Tomasi lambda_min = 0 (SURVEY O5 closed form)."""
    a, b, k = 0.25, 0.5, 0.04
    W = H = 12
    img = (a * np.arange(W)[None, :] + b * np.arange(H)[:, None]).astype(np.float32)
    s = P.harris(W, H)
    r = O.run(s, [img], [1, 2, 6, 7, 8, 9])
    inner = (slice(2, -2), slice(2, -2))
    np.testing.assert_allclose(r[1][1:-1, 1:-1], 8 * a)
    np.testing.assert_allclose(r[2][1:-1, 1:-1], 8 * b)
    np.testing.assert_allclose(r[6][inner], 64 * a * a)
    np.testing.assert_allclose(r[8][inner], 64 * a * b)
    np.testing.assert_allclose(r[9][inner], -k * (64 * (a * a + b * b)) ** 2, rtol=1e-12)
    st = O.run(P.harris(W, H, shitomasi=True), [img])
    np.testing.assert_allclose(list(st.values())[0][inner], 0.0, atol=1e-12)


@pytest.mark.parametrize("mode", ["clamp", "mirror", "mirror101", "repeat"])
def test_harris_constant_image_is_zero(mode):
    """A constant image has zero gradient everywhere under value-preserving borders."""
    img = np.full((10, 13), 0.375, np.float32)
    out = list(O.run(P.harris(13, 10, mode), [img]).values())[0]
    assert np.all(out == 0.0)


def test_harris_corner_response_sign():
    """An ideal corner gives R > 0, an edge R < 0, flat R = 0 (Harris' classification)."""
    img = np.zeros((16, 16), np.float32)
    img[8:, 8:] = 1.0
    out = list(O.run(P.harris(16, 16), [img]).values())[0]
    assert out[8, 8] > 0 and out[12, 8] < 0 and out[2, 2] == 0.0


# ------------------------------------------------------ integer semantics

def test_int_blur_preserves_constant():
    """(c*256 + 128) >> 8 == c: a constant image passes every 256-normalised blur
    of deep10 unchanged."""
    for c in (0, 1, 77, 254, 255):
        img = np.full((12, 12, 4), c, np.uint8)
        s = P.deep10(12, 12)
        r = O.run(s, [img], [1, 6])
        assert np.all(r[1] == c)


def test_int_ops_floor_shift_and_saturation():
    """SHR is an arithmetic (floor) shift; stores saturate to [0,255]; LUT clamps its index."""
    p = P.Pipeline("ints", 3, 1, "u8x4")
    i = p.input()
    a = p.point("a", [i], [P.C(-3), P.SHR(1), P.C(10), P.ADD])          # floor(-1.5) + 10 = 8
    b = p.point("b", [i], [P.L(0), P.C(300), P.ADD])                    # saturates to 255
    c = p.point("c", [i], [P.C(0), P.L(0), P.SUB])                      # -x saturates to 0 (x>0)
    d = p.point("d", [i], [P.L(0), P.C(250), P.ADD, P.LUT], lut=list(range(256)))   # index clamp
    e = p.point("e", [i], [P.C(-7), P.C(2), P.DIV, P.C(10), P.ADD])      # C truncation: -3 + 10
    for x in (a, b, c, d, e):
        p.output(x)
    img = np.array([[[1, 2, 3, 4], [100, 0, 5, 9], [200, 255, 6, 7]]], np.uint8)
    r = O.run(p.spec(), [img])
    assert np.all(r[a] == 8) and np.all(r[b] == 255)
    assert np.all(r[c][img > 0] == 0) and np.all(r[c][img == 0] == 0)
    np.testing.assert_array_equal(r[d], np.minimum(img.astype(int) + 250, 255))
    assert np.all(r[e] == 7)


def test_int32_overflow_is_reported():
    p = P.Pipeline("ovf", 2, 2, "u8x4")
    i = p.input()
    o = p.point("o", [i], [P.C(1 << 20), P.C(1 << 20), P.MUL])
    p.output(o)
    with pytest.raises(RuntimeError):
        O.run(p.spec(), [np.zeros((2, 2, 4), np.uint8)])


# ------------------------------- pointwise evaluator == materialising executor

@pytest.mark.parametrize("seed", range(12))
def test_pointwise_equals_materialised(seed):
    """The recursive per-pixel evaluation (index-exchange semantics)
    equals the materialised unfused execution on random DAGs."""
    rng = random.Random(seed)
    dtype = "f32" if seed % 2 == 0 else "u8x4"
    W, H = rng.choice([(7, 5), (9, 9), (12, 4), (3, 8)])
    s = P.random_pipeline(rng, W, H, dtype, rng.randint(2, 6))
    ins = [gen.image(dtype, seed * 10 + j, W, H) for j in range(s["n_inputs"])]
    if dtype == "u8x4":
        ins = [x for x in ins]
    full = O.run(s, ins)
    ys, xs = np.meshgrid(np.arange(H), np.arange(W), indexing="ij")
    for img_id, ref in full.items():
        got = O.eval_points(s, ins, img_id, ys.ravel(), xs.ravel())
        if dtype == "f32":
            np.testing.assert_allclose(got.reshape(H, W), ref, rtol=1e-12, atol=1e-12)
        else:
            np.testing.assert_array_equal(got.reshape(H, W, 4), ref)


def test_generator_properties():
    """Counter-based generator: band slices equal the full image; f32 in [0,1) on the 2^-24 grid."""
    full = gen.image_f32(5, 33, 17)
    band = gen.image_f32(5, 33, 17, 4, 9)
    np.testing.assert_array_equal(full[4:9], band)
    assert full.min() >= 0 and full.max() < 1
    assert np.all(full * 2 ** 24 == np.floor(full * 2 ** 24))
    u = gen.image_u8x4(5, 33, 17)
    assert u.shape == (17, 33, 4) and u.dtype == np.uint8
    assert len(np.unique(u)) > 200

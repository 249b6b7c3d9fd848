"""Seeded, counter-based synthetic image generator (SplitMix64 on the pixel index).

This module is the ONLY code shared by the oracle side and the CUDA side: it
holds no arithmetic of the method (no stencil, no fusion, no border logic),
only the random numbers that stand in for the paper's "random images"
(artifact appendix: the binaries generate random input
images).  Recipe:

    h(seed, i) = splitmix64_finalizer((seed << 40) + i + golden)     i = y*W + x
    f32   : (h >> 40) * 2**-24            uniform in [0, 1), exactly representable
    u8x4  : the 4 low bytes of (h >> 32)  (R, G, B, A) little-endian

Because the value depends only on (seed, global pixel index), a row band of a
large image can be generated on its own (multi-GPU bands, sampled parity).
"""
from __future__ import annotations

import numpy as np

_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def splitmix64(v: np.ndarray) -> np.ndarray:
    """SplitMix64 finalizer, vectorised over uint64 (wrap-around arithmetic)."""
    with np.errstate(over="ignore"):
        z = v + _GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def _hash_rows(seed: int, width: int, row0: int, row1: int) -> np.ndarray:
    idx = np.arange(row0 * width, row1 * width, dtype=np.uint64)
    with np.errstate(over="ignore"):
        base = np.uint64(seed) << np.uint64(40)
        return splitmix64(idx + base).reshape(row1 - row0, width)


def image_f32(seed: int, width: int, height: int, row0: int = 0, row1: int | None = None) -> np.ndarray:
    """float32 gray image (rows [row0, row1) of the full W x H image), values in [0, 1)."""
    row1 = height if row1 is None else row1
    h = _hash_rows(seed, width, row0, row1)
    return ((h >> np.uint64(40)).astype(np.float64) * 2.0 ** -24).astype(np.float32)


def image_u8x4(seed: int, width: int, height: int, row0: int = 0, row1: int | None = None) -> np.ndarray:
    """uint8 RGBA image, shape (rows, W, 4), interleaved channels."""
    row1 = height if row1 is None else row1
    h = _hash_rows(seed, width, row0, row1)
    lo = (h >> np.uint64(32)).astype(np.uint32)
    return lo.view(np.uint8).reshape(row1 - row0, width, 4).copy()


def image(dtype: str, seed: int, width: int, height: int, row0: int = 0, row1: int | None = None) -> np.ndarray:
    if dtype == "f32":
        return image_f32(seed, width, height, row0, row1)
    if dtype == "u8x4":
        return image_u8x4(seed, width, height, row0, row1)
    raise ValueError(f"unknown dtype {dtype!r}")

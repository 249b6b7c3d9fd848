"""TEST INFRASTRUCTURE ONLY -- Python adapter for the C oracle (kf_oracle.c).

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
--impl reference) may import this module.  The product path
(paper_conf_cgo_qiaorht19_b200/) never imports it and shares no code with it.

run(spec, inputs, ids)          -> unfused materialising execution
eval_points(spec, inputs, id, ys, xs) -> recursive pointwise evaluation (same
                                   definition; index-exchange semantics,
                                   PAPER.md:1088-1133)
border(p, n, mode)              -> the border index map
set_threads(n)                  -> OpenMP threads over rows (1 = serial)
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "kf_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

# op-IR opcode numbers, restated from the interface (include/kfuse.h kf_opcode)
OPCODES = {"LOAD": 0, "CONST": 1, "ADD": 2, "SUB": 3, "MUL": 4, "DIV": 5, "MIN": 6, "MAX": 7, "ABS": 8,
           "NEG": 9, "SQRT": 10, "EXP": 11, "LOG": 12, "POW": 13, "SHR": 14, "SHL": 15, "SAT_U8": 16,
           "CLAMP": 17, "SELECT_GT": 18, "LUT": 19}
MODES = {"clamp": 0, "mirror": 1, "mirror101": 2, "repeat": 3, "constant": 4}


class OrOp(C.Structure):
    _fields_ = [("kind", C.c_int), ("n_inputs", C.c_int), ("inputs", C.POINTER(C.c_int)),
                ("n_prog", C.c_int), ("prog_op", C.POINTER(C.c_int)), ("prog_arg", C.POINTER(C.c_int)),
                ("prog_imm", C.POINTER(C.c_double)), ("lut", C.POINTER(C.c_int)), ("lut_len", C.c_int),
                ("mw", C.c_int), ("mh", C.c_int), ("mask", C.POINTER(C.c_double)), ("mode", C.c_int),
                ("constant", C.c_double)]


def build(force: bool = False) -> str:
    """Compile the oracle (plain C, -O2 -ffp-contract=off).  Building the checker
    is not using it (__graft_entry__.build() calls this)."""
    with _lock:
        if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
            tmp = _LIB + f".{os.getpid()}.tmp"
            subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fopenmp", "-fPIC", "-shared",
                                   "-std=c11", "-o", tmp, _SRC, "-lm"])
            os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = C.CDLL(build())
        lib.or_run.restype = C.c_int
        lib.or_eval_points.restype = C.c_int
        lib.or_border.restype = C.c_int
        lib.or_border.argtypes = [C.c_int, C.c_int, C.c_int]
        lib.or_set_threads.restype = C.c_int
        lib.or_set_threads.argtypes = [C.c_int]
        # default: all cores (rows of each kernel split over threads; no arithmetic change),
        # or $KF_ORACLE_THREADS
        lib.or_set_threads(int(os.environ.get("KF_ORACLE_THREADS", "0")))
        _lib = lib
    return _lib


def set_threads(n: int) -> int:
    """Threads used by run()/eval_points(): 1 = the serial loop, <= 0 = all cores.
    Returns the number actually used."""
    return int(_load().or_set_threads(int(n)))


def border(p: int, n: int, mode: str) -> int:
    """Border index map; -1 means 'use the constant'."""
    return _load().or_border(int(p), int(n), MODES[mode])


class _Ops:
    """Keeps the ctypes arrays alive while the C call runs."""

    def __init__(self, spec: dict):
        self.keep = []
        ops = spec["ops"]
        self.arr = (OrOp * max(1, len(ops)))()
        for k, o in enumerate(ops):
            s = self.arr[k]
            s.kind = 0 if o["kind"] == "point" else 1
            s.n_inputs = len(o["inputs"])
            s.inputs = self._ints(o["inputs"])
            prog = o["prog"] if o["kind"] == "point" else o["post"]
            s.n_prog = len(prog)
            s.prog_op = self._ints([OPCODES[t[0]] for t in prog])
            s.prog_arg = self._ints([int(t[1]) for t in prog])
            s.prog_imm = self._dbls([float(t[2]) for t in prog])
            lut = o.get("lut")
            s.lut = self._ints(lut or [0])
            s.lut_len = len(lut or [])
            if o["kind"] == "local":
                m = o["mask"]
                s.mh, s.mw = len(m), len(m[0])
                s.mask = self._dbls([v for r in m for v in r])
                s.mode = MODES[o["mode"]]
                s.constant = float(o["constant"])

    def _ints(self, v):
        a = (C.c_int * max(1, len(v)))(*[int(x) for x in v])
        self.keep.append(a)
        return a

    def _dbls(self, v):
        a = (C.c_double * max(1, len(v)))(*[float(x) for x in v])
        self.keep.append(a)
        return a


def _inputs(spec: dict, inputs) -> tuple[list, C.Array]:
    W, H = spec["width"], spec["height"]
    arrs = []
    for a in inputs:
        if spec["dtype"] == "f32":
            a = np.ascontiguousarray(a, dtype=np.float32)
            assert a.shape == (H, W)
        else:
            a = np.ascontiguousarray(a, dtype=np.uint8)
            assert a.shape == (H, W, 4)
        arrs.append(a)
    assert len(arrs) == spec["n_inputs"]
    ptrs = (C.c_void_p * max(1, len(arrs)))(*[a.ctypes.data for a in arrs])
    return arrs, ptrs


def run(spec: dict, inputs, ids=None) -> dict:
    """Unfused execution of every kernel; returns {image id: array} for `ids`
    (default: the pipeline outputs).  f32 -> float64 (H, W); u8x4 -> uint8 (H, W, 4)."""
    lib = _load()
    ids = list(spec["outputs"] if ids is None else ids)
    W, H = spec["width"], spec["height"]
    ops = _Ops(spec)
    arrs, iptr = _inputs(spec, inputs)
    outs = [np.empty((H, W), np.float64) if spec["dtype"] == "f32" else np.empty((H, W, 4), np.uint8)
            for _ in ids]
    optr = (C.c_void_p * max(1, len(outs)))(*[o.ctypes.data for o in outs])
    rid = (C.c_int * max(1, len(ids)))(*ids)
    rc = lib.or_run(C.c_int(W), C.c_int(H), C.c_int(0 if spec["dtype"] == "f32" else 1),
                    C.c_int(spec["n_inputs"]), iptr, C.c_int(len(spec["ops"])), ops.arr,
                    C.c_int(len(ids)), rid, optr)
    if rc:
        raise RuntimeError(f"oracle error {rc} ({'int32 overflow' if rc == 1 else 'bad program'})")
    return dict(zip(ids, outs))


def eval_points(spec: dict, inputs, img_id: int, ys, xs) -> np.ndarray:
    """Value of image `img_id` at points (ys[i], xs[i]) by recursive evaluation."""
    lib = _load()
    ys = np.ascontiguousarray(ys, dtype=np.int32)
    xs = np.ascontiguousarray(xs, dtype=np.int32)
    n = len(ys)
    ops = _Ops(spec)
    arrs, iptr = _inputs(spec, inputs)
    out = np.empty(n, np.float64) if spec["dtype"] == "f32" else np.empty((n, 4), np.uint8)
    rc = lib.or_eval_points(C.c_int(spec["width"]), C.c_int(spec["height"]),
                            C.c_int(0 if spec["dtype"] == "f32" else 1), C.c_int(spec["n_inputs"]), iptr,
                            C.c_int(len(spec["ops"])), ops.arr, C.c_int(img_id), C.c_int(n),
                            ys.ctypes.data_as(C.c_void_p), xs.ctypes.data_as(C.c_void_p),
                            out.ctypes.data_as(C.c_void_p))
    if rc:
        raise RuntimeError(f"oracle error {rc}")
    return out

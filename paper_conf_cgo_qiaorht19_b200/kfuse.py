"""Thin ctypes binding of libkfuse (include/kfuse.h) -- argument marshalling only.

Every step of the hot path (planning, code generation, the fused kernels) runs
inside libkfuse.so; this module only converts Python/torch objects to the
C-ABI's plain pointers.  There is no CPU fallback: if libkfuse.so is missing the
import fails loudly, and every CUDA error surfaces as KfError.
"""
from __future__ import annotations

import ctypes as C
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
_LIBPATH = os.path.join(_PKG, "libkfuse.so")

if not os.path.exists(_LIBPATH):
    raise ImportError(f"libkfuse.so not built at {_LIBPATH}: run "
                      "`python -m paper_conf_cgo_qiaorht19_b200.build` (or __graft_entry__.build())")


KF_F32, KF_U8X4 = 0, 1
DTYPES = {"f32": KF_F32, "u8x4": KF_U8X4}
MODES = {"clamp": 0, "mirror": 1, "mirror101": 2, "repeat": 3, "constant": 4}
OPCODES = {"LOAD": 0, "CONST": 1, "ADD": 2, "SUB": 3, "MUL": 4, "DIV": 5, "MIN": 6, "MAX": 7, "ABS": 8,
           "NEG": 9, "SQRT": 10, "EXP": 11, "LOG": 12, "POW": 13, "SHR": 14, "SHL": 15, "SAT_U8": 16,
           "CLAMP": 17, "SELECT_GT": 18, "LUT": 19}
STATUS = ["KF_OK", "KF_ERR_ARG", "KF_ERR_BAD_ID", "KF_ERR_HEADER", "KF_ERR_MASK", "KF_ERR_FROZEN",
          "KF_ERR_ILLEGAL_BLOCK", "KF_ERR_NVRTC", "KF_ERR_CUDA", "KF_ERR_NCCL", "KF_ERR_OOM", "KF_ERR_PROGRAM"]


class KfInstr(C.Structure):
    _fields_ = [("op", C.c_int32), ("arg", C.c_int32), ("imm", C.c_double)]


class KfCost(C.Structure):
    _fields_ = [("n_alu", C.c_int32), ("n_sfu", C.c_int32)]


class ModelParams(C.Structure):
    _fields_ = [("tg", C.c_double), ("ts", C.c_double), ("c_alu", C.c_double), ("c_sfu", C.c_double),
                ("gamma", C.c_double), ("c_mshared", C.c_double), ("phi_mode", C.c_int32),
                ("tile_w", C.c_int32), ("tile_h", C.c_int32), ("eq3_mode", C.c_int32),
                ("bw_bytes_clk", C.c_double), ("issue_lanes_clk", C.c_double), ("overlap", C.c_double)]


class KfError(RuntimeError):
    def __init__(self, status: int, msg: str):
        self.status = status
        self.name = STATUS[status] if 0 <= status < len(STATUS) else str(status)
        super().__init__(f"{self.name}: {msg}")


_P = C.c_void_p
_I32P = C.POINTER(C.c_int32)
_SIGS = {
    "kf_model_params_paper": (None, [C.POINTER(ModelParams)]),
    "kf_model_params_b200": (None, [C.POINTER(ModelParams)]),
    "kf_model_params_b200_roofline": (None, [C.POINTER(ModelParams)]),
    "kf_pipeline_create": (C.c_int, [C.c_int32, C.c_int32, C.c_int, C.POINTER(_P)]),
    "kf_pipeline_destroy": (None, [_P]),
    "kf_add_input": (C.c_int, [_P, _I32P]),
    "kf_add_point_op": (C.c_int, [_P, _I32P, C.c_int32, C.POINTER(KfInstr), C.c_int32, C.POINTER(KfCost),
                                  _I32P, C.c_int32, _I32P]),
    "kf_add_local_op": (C.c_int, [_P, C.c_int32, C.POINTER(C.c_double), C.c_int32, C.c_int32, C.c_int,
                                  C.c_double, C.POINTER(KfInstr), C.c_int32, C.POINTER(KfCost), _I32P]),
    "kf_mark_output": (C.c_int, [_P, C.c_int32]),
    "kf_plan_fusion": (C.c_int, [_P, C.POINTER(ModelParams), C.POINTER(_P)]),
    "kf_plan_basic": (C.c_int, [_P, C.POINTER(ModelParams), C.POINTER(_P)]),
    "kf_peer_signal": (C.c_int, [_P, C.c_int32, _P, _P]),
    "kf_peer_pull": (C.c_int, [C.c_int32, C.c_int32, _P, _P, _P, _P, _P, _P, _P, C.c_int64, _P]),
    "kf_peer_wait": (C.c_int, [C.c_int32, _P, _P, _P, C.c_int64, _P]),
    "kf_peer_enable": (C.c_int, [C.c_int32, C.c_int32]),
    "kf_plan_exact": (C.c_int, [_P, C.POINTER(ModelParams), C.POINTER(_P)]),
    "kf_plan_unfused": (C.c_int, [_P, C.POINTER(_P)]),
    "kf_plan_from_blocks": (C.c_int, [_P, _I32P, C.POINTER(_P)]),
    "kf_plan_destroy": (None, [_P]),
    "kf_plan_num_blocks": (C.c_int32, [_P]),
    "kf_plan_block": (C.c_int, [_P, C.c_int32, _I32P, _I32P]),
    "kf_plan_objective": (C.c_int, [_P, C.POINTER(C.c_int64), C.POINTER(C.c_int64)]),
    "kf_plan_edge": (C.c_int, [_P, C.c_int32, C.c_int32, C.POINTER(C.c_double), _I32P, _I32P, _I32P]),
    "kf_plan_num_cuts": (C.c_int32, [_P]),
    "kf_plan_cut": (C.c_int, [_P, C.c_int32, _I32P, _I32P, C.POINTER(C.c_int64), C.POINTER(C.c_int64), _I32P]),
    "kf_plan_num_launches": (C.c_int32, [_P]),
    "kf_plan_halo_rows": (C.c_int32, [_P]),
    "kf_plan_kernel_source": (C.c_int, [_P, _P, C.c_int32, C.c_char_p, C.c_size_t, C.POINTER(C.c_size_t)]),
    "kf_compile_plan": (C.c_int, [_P, _P]),
    "kf_prepare": (C.c_int, [_P, _P]),
    "kf_run": (C.c_int, [_P, _P, C.POINTER(_P), C.c_int32, C.POINTER(_P), C.c_int32, _P]),
    "kf_run_host": (C.c_int, [_P, _P, C.POINTER(_P), C.c_int32, C.POINTER(_P), C.c_int32, _P]),
    "kf_bounds_report": (C.c_int, [_P, C.POINTER(C.c_int64), C.POINTER(C.c_uint64), C.POINTER(C.c_int32)]),
    "kf_run_host_async": (C.c_int, [_P, _P, C.POINTER(_P), C.c_int32, C.POINTER(_P), C.c_int32, _P]),
    "kf_run_batch": (C.c_int, [_P, _P, C.c_int32, C.POINTER(_P), C.c_int32, C.POINTER(_P), C.c_int32, _P]),
    "kf_run_band": (C.c_int, [_P, _P, C.c_int32, C.c_int32, C.POINTER(_P), C.c_int32, C.c_int32,
                              C.POINTER(_P), _P]),
    "kf_set_option": (C.c_int, [_P, C.c_char_p, C.c_int64]),
    "kf_get_option": (C.c_int, [_P, C.c_char_p, C.POINTER(C.c_int64)]),
    "kf_last_error": (C.c_char_p, []),
    "kf_version": (C.c_char_p, []),
}


def _open(path: str) -> C.CDLL:
    """Loads a libkfuse build and declares the C-ABI signatures."""
    lb = C.CDLL(path)
    for n, (r, a) in _SIGS.items():
        f = getattr(lb, n)
        f.restype = r
        f.argtypes = a
    return lb


lib = _open(_LIBPATH)

EXPORTED = sorted(_SIGS)


def _check(st: int) -> None:
    if st != 0:
        raise KfError(st, lib.kf_last_error().decode(errors="replace"))


def model_params(profile: str = "paper", **over) -> ModelParams:
    m = ModelParams()
    {"b200": lib.kf_model_params_b200, "b200roof": lib.kf_model_params_b200_roofline}.get(
        profile, lib.kf_model_params_paper)(C.byref(m))
    for k, v in over.items():
        setattr(m, k, v)
    return m


def _prog(prog) -> tuple:
    arr = (KfInstr * max(1, len(prog)))()
    for i, (name, arg, imm) in enumerate(prog):
        arr[i].op, arr[i].arg, arr[i].imm = OPCODES[name], int(arg), float(imm)
    return arr, len(prog)


def _ptrs(vals) -> C.Array:
    return (_P * max(1, len(vals)))(*[_P(int(v)) for v in vals])


def _dptr(t) -> int:
    """Device/host address of a torch tensor, numpy array or int."""
    if isinstance(t, int):
        return t
    if hasattr(t, "data_ptr"):
        return t.data_ptr()
    return t.ctypes.data


class Pipeline:
    """kf_pipeline: a kernel DAG over one W x H iteration space."""

    def __init__(self, width: int, height: int, dtype: str = "f32"):
        self.width, self.height, self.dtype = int(width), int(height), dtype
        h = _P()
        _check(lib.kf_pipeline_create(self.width, self.height, DTYPES[dtype], C.byref(h)))
        self.h = h
        self.n_inputs = 0
        self.n_kernels = 0
        self.outputs: list[int] = []

    def __del__(self):
        if getattr(self, "h", None) and lib is not None:
            lib.kf_pipeline_destroy(self.h)
            self.h = None

    def add_input(self) -> int:
        i = C.c_int32()
        _check(lib.kf_add_input(self.h, C.byref(i)))
        self.n_inputs += 1
        return i.value

    def add_point_op(self, inputs, prog, cost=None, lut=None) -> int:
        ins = (C.c_int32 * len(inputs))(*inputs)
        arr, n = _prog(prog)
        c = C.byref(KfCost(*cost)) if cost is not None else None
        lt = (C.c_int32 * len(lut))(*lut) if lut is not None else None
        out = C.c_int32()
        _check(lib.kf_add_point_op(self.h, ins, len(inputs), arr, n, c, lt, len(lut) if lut else 0,
                                   C.byref(out)))
        self.n_kernels += 1
        return out.value

    def add_local_op(self, inp, mask, mode="clamp", constant=0.0, post=None, cost=None) -> int:
        mh, mw = len(mask), len(mask[0])
        flat = (C.c_double * (mw * mh))(*[float(v) for r in mask for v in r])
        arr, n = _prog(post or [])
        c = C.byref(KfCost(*cost)) if cost is not None else None
        out = C.c_int32()
        _check(lib.kf_add_local_op(self.h, int(inp), flat, mw, mh, MODES[mode], float(constant), arr, n, c,
                                   C.byref(out)))
        self.n_kernels += 1
        return out.value

    def mark_output(self, img: int) -> None:
        _check(lib.kf_mark_output(self.h, int(img)))
        self.outputs.append(int(img))

    def set_option(self, name: str, value: int) -> None:
        """kf_set_option: a schedule option (results are bit-identical for every value)."""
        _check(lib.kf_set_option(self.h, name.encode(), int(value)))

    def get_option(self, name: str) -> int:
        v = C.c_int64()
        _check(lib.kf_get_option(self.h, name.encode(), C.byref(v)))
        return v.value

    @classmethod
    def from_spec(cls, spec: dict, options: dict | None = None) -> "Pipeline":
        """Builds the pipeline of a plain-data description (kf_inputs.pipelines),
        with optional schedule options {name: value}."""
        p = cls(spec["width"], spec["height"], spec["dtype"])
        for name, value in (options or {}).items():
            p.set_option(name, value)
        for _ in range(spec["n_inputs"]):
            p.add_input()
        for o in spec["ops"]:
            if o["kind"] == "point":
                p.add_point_op(o["inputs"], o["prog"], o.get("cost"), o.get("lut"))
            else:
                p.add_local_op(o["inputs"][0], o["mask"], o["mode"], o["constant"], o["post"], o.get("cost"))
        for img in spec["outputs"]:
            p.mark_output(img)
        return p

    # ---- planning
    def plan_fusion(self, profile="paper", **over) -> "Plan":
        m = model_params(profile, **over) if isinstance(profile, str) else profile
        h = _P()
        _check(lib.kf_plan_fusion(self.h, C.byref(m), C.byref(h)))
        return Plan(self, h)

    def plan_basic(self, profile="paper", **over) -> "Plan":
        """kf_plan_basic: the basic fusion of [12] (comparison column of Table I)."""
        m = model_params(profile, **over) if isinstance(profile, str) else profile
        h = _P()
        _check(lib.kf_plan_basic(self.h, C.byref(m), C.byref(h)))
        return Plan(self, h)

    def plan_exact(self, profile="paper", **over) -> "Plan":
        """kf_plan_exact: the optimum of Eq. 1 over all legal partitions (<= 16 kernels)."""
        m = model_params(profile, **over) if isinstance(profile, str) else profile
        h = _P()
        _check(lib.kf_plan_exact(self.h, C.byref(m), C.byref(h)))
        return Plan(self, h)

    def plan_unfused(self) -> "Plan":
        h = _P()
        _check(lib.kf_plan_unfused(self.h, C.byref(h)))
        return Plan(self, h)

    def plan_from_blocks(self, block_of_kernel) -> "Plan":
        arr = (C.c_int32 * len(block_of_kernel))(*block_of_kernel)
        h = _P()
        _check(lib.kf_plan_from_blocks(self.h, arr, C.byref(h)))
        return Plan(self, h)


class Plan:
    """kf_plan: a partition of the kernels into fused blocks, plus compiled kernels."""

    def __init__(self, pipe: Pipeline, h):
        self.pipe, self.h = pipe, h

    def __del__(self):
        if getattr(self, "h", None) and lib is not None:
            lib.kf_plan_destroy(self.h)
            self.h = None

    @property
    def blocks(self) -> list[list[int]]:
        out = []
        for i in range(lib.kf_plan_num_blocks(self.h)):
            n = C.c_int32()
            buf = (C.c_int32 * 64)()
            _check(lib.kf_plan_block(self.h, i, buf, C.byref(n)))
            out.append(list(buf[: n.value]))
        return out

    @property
    def objective(self) -> tuple[int, int]:
        q, e = C.c_int64(), C.c_int64()
        _check(lib.kf_plan_objective(self.h, C.byref(q), C.byref(e)))
        return q.value, e.value

    def edge(self, src: int, dst: int) -> dict:
        w, eps, leg, prof = C.c_double(), C.c_int32(), C.c_int32(), C.c_int32()
        _check(lib.kf_plan_edge(self.h, src, dst, C.byref(w), C.byref(eps), C.byref(leg), C.byref(prof)))
        return {"w": w.value, "is_eps": bool(eps.value), "ctx_legal": bool(leg.value),
                "profitable": bool(prof.value)}

    @property
    def cuts(self) -> list[tuple]:
        out = []
        for i in range(lib.kf_plan_num_cuts(self.h)):
            buf = (C.c_int32 * 64)()
            n, q, e, ph = C.c_int32(), C.c_int64(), C.c_int64(), C.c_int32()
            _check(lib.kf_plan_cut(self.h, i, buf, C.byref(n), C.byref(q), C.byref(e), C.byref(ph)))
            out.append((list(buf[: n.value]), (q.value, e.value), ph.value))
        return out

    @property
    def num_launches(self) -> int:
        return lib.kf_plan_num_launches(self.h)

    @property
    def halo_rows(self) -> int:
        return lib.kf_plan_halo_rows(self.h)

    def source(self, block: int) -> str:
        n = C.c_size_t()
        _check(lib.kf_plan_kernel_source(self.pipe.h, self.h, block, None, 0, C.byref(n)))
        buf = C.create_string_buffer(n.value + 1)
        _check(lib.kf_plan_kernel_source(self.pipe.h, self.h, block, buf, n.value + 1, C.byref(n)))
        return buf.value.decode()

    def compile(self) -> None:
        """NVRTC-compile every block into the cubin cache (no GPU needed)."""
        _check(lib.kf_compile_plan(self.pipe.h, self.h))

    def prepare(self) -> None:
        _check(lib.kf_prepare(self.pipe.h, self.h))

    def run(self, inputs, outputs, stream=None) -> None:
        """inputs/outputs: CUDA tensors (or raw device addresses), dense, 16-B aligned.
        stream: a torch.cuda.Stream, a raw cudaStream_t int, or None = torch's current stream."""
        _check(lib.kf_run(self.pipe.h, self.h, _ptrs([_dptr(t) for t in inputs]), len(inputs),
                          _ptrs([_dptr(t) for t in outputs]), len(outputs), _P(_stream(stream))))

    def run_batch(self, frames_in, frames_out, stream=None) -> None:
        """Independent frames (kf_run_batch): frames_in[f] / frames_out[f] are the
        input / output lists of frame f, as for run()."""
        n = len(frames_in)
        if len(frames_out) != n:
            raise ValueError("frames_in and frames_out differ in length")
        n_in = len(frames_in[0]) if n else self.pipe.n_inputs
        n_out = len(frames_out[0]) if n else 0
        if any(len(f) != n_in for f in frames_in) or any(len(f) != n_out for f in frames_out):
            raise ValueError("every frame needs the same number of inputs and outputs")
        _check(lib.kf_run_batch(self.pipe.h, self.h, n,
                                _ptrs([_dptr(t) for f in frames_in for t in f]), n_in,
                                _ptrs([_dptr(t) for f in frames_out for t in f]), n_out, _P(_stream(stream))))

    def run_host(self, inputs, outputs, stream=None) -> None:
        """End-to-end: host numpy/pinned-tensor buffers in and out (kf_run_host)."""
        _check(lib.kf_run_host(self.pipe.h, self.h, _ptrs([_dptr(t) for t in inputs]), len(inputs),
                               _ptrs([_dptr(t) for t in outputs]), len(outputs), _P(_stream(stream))))

    def run_host_async(self, inputs, outputs, stream=None) -> None:
        """kf_run_host_async: pinned host buffers; no final synchronisation."""
        _check(lib.kf_run_host_async(self.pipe.h, self.h, _ptrs([_dptr(t) for t in inputs]), len(inputs),
                                     _ptrs([_dptr(t) for t in outputs]), len(outputs), _P(_stream(stream))))

    def run_band(self, row0, row1, in_band, in_row0, in_row1, out_band, stream=None) -> None:
        _check(lib.kf_run_band(self.pipe.h, self.h, int(row0), int(row1),
                               _ptrs([_dptr(t) for t in in_band]), int(in_row0), int(in_row1),
                               _ptrs([_dptr(t) for t in out_band]), _P(_stream(stream))))


def _stream(stream) -> int:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def _i64s(vals) -> C.Array:
    return (C.c_int64 * max(1, len(vals)))(*[int(v) for v in vals])


def peer_signal(flags, sent=0, stream=None) -> None:
    """kf_peer_signal: release-increment counters (device addresses, may be peer)."""
    _check(lib.kf_peer_signal(_ptrs(flags), len(flags), _P(int(sent)), _P(_stream(stream))))


def peer_pull(dst, src, nbytes, flag, seen, ack, err, spin_limit=1 << 27, stream=None, copies=1) -> None:
    """kf_peer_pull over len(flag) segments of `copies` copies each (dst/src/nbytes
    hold len(flag) * copies entries, segment-major; all arguments device
    addresses; ack entries may be 0)."""
    _check(lib.kf_peer_pull(len(flag), int(copies), _ptrs(dst), _ptrs(src), _i64s(nbytes), _ptrs(flag),
                            _ptrs(seen), _ptrs(ack), _P(int(err)), int(spin_limit), _P(_stream(stream))))


def peer_wait(counter, target, err, spin_limit=1 << 27, stream=None) -> None:
    """kf_peer_wait: wait until every counter[i] reaches target[i] (device addresses)."""
    _check(lib.kf_peer_wait(len(counter), _ptrs(counter), _ptrs(target), _P(int(err)), int(spin_limit),
                            _P(_stream(stream))))


def peer_enable(device: int, peer_device: int) -> None:
    """kf_peer_enable: kernels on `device` may access `peer_device`'s memory."""
    _check(lib.kf_peer_enable(int(device), int(peer_device)))


def bounds_report(pipe: "Pipeline") -> tuple[int, int, int]:
    """kf_bounds_report (bounds-checking build only): (violations, first address, kind)."""
    n, ad, k = C.c_int64(), C.c_uint64(), C.c_int32()
    _check(lib.kf_bounds_report(pipe.h, C.byref(n), C.byref(ad), C.byref(k)))
    return n.value, ad.value, k.value


def version() -> str:
    return lib.kf_version().decode()

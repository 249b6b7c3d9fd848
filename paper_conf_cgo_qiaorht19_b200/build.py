"""Builds libkfuse.so in-tree with nvcc for sm_100a (no GPU needed).

    python -m paper_conf_cgo_qiaorht19_b200.build [--force]

The device header csrc/device/kf_device.cuh is embedded into the library as a
string (it is handed to NVRTC for every generated block kernel).
"""
from __future__ import annotations

import hashlib
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(PKG, "build")
LIB = os.path.join(PKG, "libkfuse.so")
ROOT = os.path.dirname(PKG)
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC,-Wall",
         "-I", os.path.join(ROOT, "include"), "-I", CSRC]
SOURCES = ["capi.cpp", "graph.cpp", "planner.cpp", "codegen.cpp", "runtime.cu", "peer.cu"]


def _embed_header() -> str:
    src = os.path.join(CSRC, "device", "kf_device.cuh")
    out = os.path.join(CSRC, "kf_device_cuh.inc")
    with open(src) as f:
        text = f.read()
    body = 'R"KFDEV(' + text + ')KFDEV"\n'
    if not os.path.exists(out) or open(out).read() != body:
        with open(out, "w") as f:
            f.write(body)
    return out


def _digest(paths) -> str:
    h = hashlib.sha256()
    for p in paths:
        with open(p, "rb") as f:
            h.update(f.read())
    h.update(" ".join(ARCH + FLAGS).encode())
    return h.hexdigest()


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    _embed_header()
    headers = [os.path.join(CSRC, "kf_internal.h"), os.path.join(CSRC, "kf_device_cuh.inc"),
               os.path.join(ROOT, "include", "kfuse.h")]
    objs = []
    for s in SOURCES:
        src = os.path.join(CSRC, s)
        obj = os.path.join(BUILD, s + ".o")
        stamp = obj + ".sha"
        dig = _digest([src] + headers)
        objs.append(obj)
        if not force and os.path.exists(obj) and os.path.exists(stamp) and open(stamp).read() == dig:
            continue
        cmd = [NVCC] + ARCH + FLAGS + ["-c", src, "-o", obj]
        if s.endswith(".cpp"):
            cmd = [NVCC] + ARCH + FLAGS + ["-x", "cu", "-c", src, "-o", obj]
        if verbose:
            print(" ".join(cmd))
        subprocess.check_call(cmd)
        with open(stamp, "w") as f:
            f.write(dig)
    tmp = LIB + f".{os.getpid()}.tmp"
    cmd = [NVCC] + ARCH + ["-shared", "-o", tmp] + objs + [
        "-L/usr/local/cuda/lib64", "-lnvrtc", "-lcudart_static", "-ldl", "-lrt", "-lpthread",
        "-Xlinker", "-rpath=/usr/local/cuda/lib64"]
    if verbose:
        print(" ".join(cmd))
    subprocess.check_call(cmd)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)

"""SASS summary of the fused kernels (no GPU needed): compiles the B200-profile
plan of each config (with optional schedule options) into a private cubin cache
and prints, per kernel, the registers / stack / shared memory, the counts of
the memory-path instructions that prove the feed (LDGSTS = cp.async, UBLKCP =
TMA bulk copy, SYNCS = mbarrier, LDS/STG.E.128) and the instruction mix of the
hottest streaming loop (the largest backward-branch body with warp shuffles).

    python tools/sass_summary.py C3 C3s C2 C4 C4:rtrip=1 C3:tma=1 > profiles/r02_sass_summary.txt
"""
import os
import re
import subprocess
import sys
import tempfile
from collections import Counter

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def cubin_for(cfg: str, opts: dict) -> str:
    d = tempfile.mkdtemp(prefix="kfsass_")
    code = ("import sys; sys.path.insert(0, %r)\n"
            "from kf_inputs import pipelines as P\n"
            "from paper_conf_cgo_qiaorht19_b200 import kfuse as K\n"
            "spec, _ = P.config(%r)\n"
            "K.Pipeline.from_spec(spec, %r).plan_fusion('b200').compile()\n") % (ROOT, cfg, opts)
    subprocess.run([sys.executable, "-c", code], check=True, env=dict(os.environ, KFUSE_CACHE_DIR=d))
    z = os.path.join(d, [f for f in os.listdir(d) if f.endswith(".cubin.z")][0])
    return plain_cubin(z)


def plain_cubin(path: str) -> str:
    """A cache entry ("KFZ1", u64 size, zlib stream) decompressed next to it."""
    import zlib
    with open(path, "rb") as f:
        z = f.read()
    out = path[:-2] if path.endswith(".z") else path + ".cubin"
    with open(out, "wb") as f:
        f.write(zlib.decompress(z[12:]))
    return out


def summary(path: str) -> str:
    sass = subprocess.run(["cuobjdump", "-sass", path], capture_output=True, text=True).stdout
    res = subprocess.run(["cuobjdump", "-res-usage", path], capture_output=True, text=True).stdout
    regs = re.search(r"REG:(\d+) STACK:(\d+) SHARED:(\d+)", res)
    ins = []
    for line in sass.splitlines():
        m = re.match(r"\s*/\*([0-9a-f]+)\*/\s*(.*?);", line)
        if m:
            ins.append((int(m.group(1), 16), m.group(2)))
    ops = Counter([x for x in t.split() if not x.startswith("@")][0] for _, t in ins)
    feed = {k: v for k, v in ops.items() if re.match(r"(LDGSTS|UBLKCP|UTMALDG|SYNCS|LDS|STG|LDG|DEPBAR)", k)}
    loops = []
    for a, t in ins:
        m = re.search(r"BRA\s*(?:!?U?P\d,\s*)?0x([0-9a-f]+)", t)
        if m and int(m.group(1), 16) < a:
            s = int(m.group(1), 16)
            body = [t2 for a2, t2 in ins if s <= a2 <= a]
            if any("SHFL" in t2 for t2 in body) and len(body) < 8000:
                loops.append(body)
    out = [f"  regs {regs.group(1)}  stack {regs.group(2)} B  smem {regs.group(3)} B  total SASS {len(ins)}",
           f"  memory-path instructions (whole kernel): {dict(sorted(feed.items()))}"]
    if loops:
        body = max(loops, key=len)
        c = Counter([x for x in t.split() if not x.startswith("@")][0] for t in body)
        out.append(f"  hottest streaming loop: {len(body)} instructions; mix {c.most_common(18)}")
    return "\n".join(out)


if __name__ == "__main__":
    for arg in sys.argv[1:]:
        cfg, _, o = arg.partition(":")
        opts = {k: int(v) for k, v in (kv.split("=") for kv in o.split(",") if kv)}
        print(f"{cfg} b200 plan, options {opts or 'default'}")
        print(summary(cubin_for(cfg, opts)))

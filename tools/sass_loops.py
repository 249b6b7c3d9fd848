"""Instruction mix of the streaming loops of a cubin (diagnostics): every
backward branch whose body holds warp shuffles, largest first.

    python tools/sass_loops.py <file.cubin | kcache/*.cubin.z> [n]
"""
import re
import subprocess
import sys
from collections import Counter

path = sys.argv[1]
if path.endswith(".z"):   # a kcache entry: "KFZ1", u64 size, zlib stream
    import tempfile
    import zlib
    with open(path, "rb") as f:
        raw = zlib.decompress(f.read()[12:])
    path = tempfile.mktemp(suffix=".cubin")
    with open(path, "wb") as f:
        f.write(raw)
sass = subprocess.run(["cuobjdump", "-sass", path], capture_output=True, text=True).stdout
ins = []
for line in sass.splitlines():
    m = re.match(r"\s*/\*([0-9a-f]+)\*/\s*(.*?);", line)
    if m:
        ins.append((int(m.group(1), 16), m.group(2)))
loops = []
for a, t in ins:
    m = re.search(r"BRA\s*(?:!?U?P\d,\s*)?0x([0-9a-f]+)", t)
    if m and int(m.group(1), 16) < a:
        loops.append((int(m.group(1), 16), a))
for s, e in loops:
    c = Counter()
    for a, t in ins:
        if s <= a <= e:
            c[[x for x in t.split() if not x.startswith("@")][0]] += 1
    if c["SHFL.UP"] + c["SHFL.DOWN"]:
        print(hex(s), hex(e), sum(c.values()), c.most_common(int(sys.argv[2]) if len(sys.argv) > 2 else 16))

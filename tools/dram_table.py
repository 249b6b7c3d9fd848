"""Summarises the ncu DRAM captures (tools/gpu_r2x.sh) into a markdown table:
measured DRAM bytes per pixel per plan (sum over the plan's launches of one run,
cold L2: --cache-control all) against the algorithmic bytes of SURVEY §8(d)."""
import csv
import collections
import glob
import os
import sys

PX = {"C2": 2048 * 2048, "C3": 4096 * 4096, "C3s": 4096 * 4096, "C4": 7680 * 4320}
ALG = {"C3": {"unfused": 84, "paper": 60, "b200": 8}, "C3s": {"unfused": 84, "paper": 60, "b200": 8},
       "C2": {"unfused": 44, "paper": 8, "b200": 8}, "C4": {"unfused": 100, "paper": 92, "b200": 8}}


def load(path):
    rows = list(csv.reader(open(path)))
    hdr, data = None, []
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            data.append(dict(zip(hdr, r)))
    per = collections.defaultdict(dict)
    for d in data:
        v = float(d["Metric Value"].replace(",", ""))
        unit = d["Metric Unit"]
        if unit in ("Mbyte", "MB"):
            v *= 1e6
        elif unit in ("Kbyte", "KB"):
            v *= 1e3
        elif unit in ("Gbyte", "GB"):
            v *= 1e9
        elif unit in ("usecond", "us"):
            v *= 1e-6
        elif unit in ("msecond", "ms"):
            v *= 1e-3
        elif unit in ("nsecond", "ns"):
            v *= 1e-9
        per[int(d["ID"])][d["Metric Name"]] = v
        per[int(d["ID"])]["name"] = d["Kernel Name"]
    return per


def main(d):
    out = ["| cfg | plan | launches / run | DRAM read B/px | DRAM write B/px | DRAM total B/px | algorithmic B/px | L2 B/px | kernel µs (cold, serialised) |",
           "|---|---|---|---|---|---|---|---|---|"]
    for cfg in ("C3", "C3s", "C2", "C4"):
        for plan in ("unfused", "paper", "b200"):
            f = os.path.join(d, f"dram_{cfg}_{plan}.csv")
            if not os.path.exists(f):
                continue
            per = load(f)
            ids = sorted(per)
            kern = [i for i in ids if per[i]["name"].startswith("kf_")]
            if not kern:
                continue
            # the runs are identical: take the last run's launches (second half)
            n = len(kern) // 2 or len(kern)
            last = kern[-n:]
            rd = sum(per[i].get("dram__bytes_read.sum", 0) for i in last) / PX[cfg]
            wr = sum(per[i].get("dram__bytes_write.sum", 0) for i in last) / PX[cfg]
            l2 = sum(per[i].get("lts__t_bytes.sum", 0) for i in last) / PX[cfg]
            us = sum(per[i].get("gpu__time_duration.sum", 0) for i in last) * 1e6
            out.append(f"| {cfg} | {plan} | {n} | {rd:.2f} | {wr:.2f} | {rd + wr:.2f} | {ALG[cfg][plan]} | {l2:.1f} | {us:.1f} |")
    print("\n".join(out))


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out")

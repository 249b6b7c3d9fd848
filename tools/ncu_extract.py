"""Extracts the counters DESIGN.md / bench.py quote from ncu --set full reports
(diagnostics): time, DRAM bytes, instructions, registers, warps active, issue
and pipe utilisation, grid, and the top stall reasons per issue.

    python tools/ncu_extract.py C3=gpurun_out/x_C3.ncu-rep C4=gpurun_out/x_C4.ncu-rep > out.json
"""
import csv
import io
import json
import subprocess
import sys

PX = {"C2": 2048 * 2048, "C3": 4096 * 4096, "C3s": 4096 * 4096, "C4": 7680 * 4320, "C5": 16384 * 16384}
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__inst_executed.sum",
        "launch__registers_per_thread", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_elapsed", "launch__grid_size"]
STALL = "smsp__average_warps_issue_stalled_"


def raw(rep: str) -> tuple[dict, dict]:
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    head, units, vals = rows[0], rows[1], rows[2]
    return dict(zip(head, vals)), dict(zip(head, units))


def main():
    res = {}
    for arg in sys.argv[1:]:
        cfg, rep = arg.split("=", 1)
        v, u = raw(rep)
        d = {k: v.get(k) for k in KEYS}
        d["units"] = {k: u.get(k) for k in KEYS[:3]}
        st = []
        for k, x in v.items():
            if k.startswith(STALL) and k.endswith("_per_issue_active.ratio"):
                try:
                    st.append((k[len(STALL):-len("_per_issue_active.ratio")], float(x)))
                except ValueError:
                    pass
        d["stalls_per_issue"] = sorted(st, key=lambda t: -t[1])[:8]
        if cfg in PX and d["smsp__inst_executed.sum"]:
            d["warp_inst_per_px"] = float(d["smsp__inst_executed.sum"].replace(",", "")) / PX[cfg]
        d["report"] = rep
        res[cfg] = d
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()

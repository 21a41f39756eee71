#!/usr/bin/env python
"""Summarise an ncu --set full capture of rap_fused_kernel into profiles/ (dev tool).

usage: ncu_summary.py REPORT.ncu-rep OUT.txt [workload-name]
Also records dram read+write bytes per launch in profiles/traffic.json, which
bench.py reports as roofline.traffic.
"""
import csv
import io
import json
import os
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "smsp__inst_executed.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__grid_size", "launch__block_size", "launch__registers_per_thread", "launch__occupancy_limit_registers",
        "sm__cycles_active.avg", "lts__t_sectors.sum", "sass__inst_executed_local_loads",
        "smsp__pcsamp_warps_issue_stalled_long_scoreboard", "smsp__pcsamp_warps_issue_stalled_barrier",
        "smsp__pcsamp_warps_issue_stalled_wait", "smsp__pcsamp_warps_issue_stalled_short_scoreboard"]


def main():
    rep, out = sys.argv[1], sys.argv[2]
    wl = sys.argv[3] if len(sys.argv) > 3 else "criteo_terabyte_c2"
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    lines = [f"ncu --set full summary of {os.path.basename(rep)} ({len(data)} launch(es) of the captured kernel)"]
    vals = {}
    for k in KEYS:
        if k in hdr:
            i = hdr.index(k)
            vals[k] = [d[i] for d in data]
            lines.append(f"{k:60s} {units[i]:>10s}  " + "  ".join(vals[k]))
    with open(out, "w") as f:
        f.write("\n".join(lines) + "\n")
    print("\n".join(lines))

    def mb(k, u):
        x = float(vals[k][0])
        return x * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[u]
    try:
        r = mb("dram__bytes_read.sum", units[hdr.index("dram__bytes_read.sum")])
        w = mb("dram__bytes_write.sum", units[hdr.index("dram__bytes_write.sum")])
        root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
        p = os.path.join(root, "profiles", "traffic.json")
        d = json.load(open(p)) if os.path.exists(p) else {}
        d[wl] = int(r + w)
        json.dump(d, open(p, "w"), indent=1)
        # the issue roofline of the same capture (bench.py roofline.issue)
        q = os.path.join(root, "profiles", "issue.json")
        e = json.load(open(q)) if os.path.exists(q) else {}
        e[wl] = {"warp_inst_per_launch": float(vals["smsp__inst_executed.sum"][0]),
                 "issue_active_pct": float(vals["smsp__issue_active.avg.pct_of_peak_sustained_active"][0]),
                 "warps_active_pct": float(vals["sm__warps_active.avg.pct_of_peak_sustained_active"][0]),
                 "ncu_us": float(vals["gpu__time_duration.sum"][0]), "summary": "profiles/" + os.path.basename(out)}
        json.dump(e, open(q, "w"), indent=1)
    except Exception as e:  # noqa: BLE001
        print("traffic not recorded:", e)


if __name__ == "__main__":
    main()

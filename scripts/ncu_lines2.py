#!/usr/bin/env python
"""Per-source-line instructions and stall samples from an ncu report
(`--print-source cuda,sass`), summed over SASS lines (dev tool).
usage: ncu_lines2.py REPORT [TOP]"""
import csv
import io
import subprocess
import sys


def main():
    rep = sys.argv[1]
    top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
    txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    cur_file, hdr, agg, tot_i, tot_s = None, None, {}, 0.0, 0.0
    for r in csv.reader(io.StringIO(txt)):
        if not r:
            continue
        if r[0] == "File Path":
            cur_file = r[1].split("/")[-1]
            continue
        if r[0] == "Function Name":
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or len(r) != len(hdr) or r[0] == "":
            continue
        d = dict(zip(hdr[4:], r[4:]))
        try:
            ie = float(d.get("Instructions Executed") or 0)
            ws = float(d.get("Warp Stall Sampling (All Samples)") or 0)
        except ValueError:
            continue
        key = (cur_file, int(r[0]))
        a = agg.setdefault(key, [0.0, 0.0, r[1][:90]])
        a[0] += ie
        a[1] += ws
        tot_i += ie
        tot_s += ws
    print(f"total warp instructions {tot_i:.0f}, stall samples {tot_s:.0f}")
    for (f, ln), (ie, ws, src) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
        print(f"{ie:12.0f} {100 * ie / max(tot_i, 1):5.1f}% {ws:6.0f} {f}:{ln:<5d} {src.strip()}")
    print("--- by stall samples")
    for (f, ln), (ie, ws, src) in sorted(agg.items(), key=lambda kv: -kv[1][1])[:top // 2]:
        print(f"{ws:6.0f} {100 * ws / max(tot_s, 1):5.1f}% {ie:12.0f} {f}:{ln:<5d} {src.strip()}")


if __name__ == "__main__":
    main()

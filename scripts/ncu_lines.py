#!/usr/bin/env python
"""Aggregate an ncu SASS source page per CUDA source line.

usage: ncu_lines.py REPORT.ncu-rep LIB.so [kernel-substring] [top]
Maps SASS offsets to file:line with nvdisasm --print-line-info on the cubin
extracted from LIB.so and sums warp-stall samples and executed instructions.
"""
import collections
import csv
import io
import os
import re
import subprocess
import sys
import tempfile


def line_map(lib, kname):
    d = tempfile.mkdtemp()
    subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(lib)], cwd=d, capture_output=True)
    cubins = [f for f in os.listdir(d) if f.endswith(".cubin")]
    for cb in cubins:
        txt = subprocess.run(["nvdisasm", "--print-line-info", os.path.join(d, cb)], capture_output=True,
                             text=True).stdout
        sec = None
        cur = None
        m = {}
        for ln in txt.splitlines():
            if ln.startswith("//---------------------") and ".text." in ln:
                sec = ln.split(".text.")[1].split()[0]
                continue
            if sec is None or kname not in sec:
                continue
            mm = re.search(r'//## File "([^"]+)", line (\d+)', ln)
            if mm:
                cur = f"{os.path.basename(mm.group(1))}:{mm.group(2)}"
                continue
            mo = re.match(r"\s+/\*([0-9a-f]{4,})\*/", ln)
            if mo:
                m[int(mo.group(1), 16)] = cur
        if m:
            return m
    return {}


def main():
    rep, lib = sys.argv[1], sys.argv[2]
    kname = sys.argv[3] if len(sys.argv) > 3 else "rap_fused_kernelILi32ELi64"
    top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = rows[1]
    idx = {h: i for i, h in enumerate(hdr)}
    data = [r for r in rows[2:] if len(r) == len(hdr) and r[0].startswith("0x")]
    base = int(data[0][0], 16)
    lm = line_map(lib, kname)
    agg = collections.defaultdict(lambda: [0, 0, 0])
    tot = [0, 0, 0]
    for r in data:
        off = int(r[0], 16) - base
        key = lm.get(off, "?")
        s = int(r[idx["Warp Stall Sampling (All Samples)"]] or 0)
        ie = int(r[idx["Instructions Executed"]] or 0)
        te = int(r[idx["Thread Instructions Executed"]] or 0)
        for i, v in enumerate((s, ie, te)):
            agg[key][i] += v
            tot[i] += v
    print(f"total stall samples {tot[0]}, warp instr {tot[1]}, thread instr {tot[2]}")
    print(f"{'line':32s} {'stall%':>7s} {'winstr%':>8s} {'winstr':>12s}")
    for k, v in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
        print(f"{k:32s} {100 * v[0] / max(tot[0], 1):7.2f} {100 * v[1] / max(tot[1], 1):8.2f} {v[1]:12d}")
    src = os.environ.get("SRC")  # optional: per-function totals (function = last definition above the line)
    if src:
        starts = []
        for i, ln in enumerate(open(src).read().splitlines(), 1):
            m = re.match(r"^(?:__device__|__global__|template|static|[a-z_]+ )[^;{]*?([A-Za-z_0-9]+)\(", ln)
            if m and not ln.startswith("template"):
                starts.append((i, m.group(1)))
        fn = collections.defaultdict(lambda: [0, 0])
        for k, v in agg.items():
            f = "?"
            if k and k.split(":")[0] == os.environ.get("SRCNAME", os.path.basename(src)):
                n = int(k.split(":")[1])
                for i, name in starts:
                    if i <= n:
                        f = name
            elif k:
                f = k.split(":")[0]
            fn[f][0] += v[0]
            fn[f][1] += v[1]
        print(f"\n{'function':32s} {'stall%':>7s} {'winstr%':>8s}")
        for k, v in sorted(fn.items(), key=lambda kv: -kv[1][1])[:top]:
            print(f"{k:32s} {100 * v[0] / max(tot[0], 1):7.2f} {100 * v[1] / max(tot[1], 1):8.2f}")


if __name__ == "__main__":
    main()

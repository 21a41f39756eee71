#!/usr/bin/env python
"""Warp-stall samples by reason from an ncu `--page source --csv --print-source
sass` export (dev tool).  usage: stall_summary.py SASS.csv TITLE > OUT.txt"""
import csv
import sys


def main():
    rows = list(csv.reader(open(sys.argv[1])))
    hdr = rows[1]
    data = [r for r in rows[2:] if len(r) == len(hdr)]
    col = {h: i for i, h in enumerate(hdr)}
    num = lambda r, h: float(r[col[h]] or 0)
    stalls = [h for h in hdr if h.startswith("stall_") and "(Not Issued)" not in h]
    tot = {h: sum(num(r, h) for r in data) for h in stalls}
    n = sum(tot.values())
    print(sys.argv[2] if len(sys.argv) > 2 else sys.argv[1])
    print(f"warp instructions {int(sum(num(r, 'Instructions Executed') for r in data))} SASS lines {len(data)} samples {int(n)}")
    for h, v in sorted(tot.items(), key=lambda kv: -kv[1]):
        print(f"{h:<30} {int(v):6d} {100 * v / max(n, 1):5.1f}%")


if __name__ == "__main__":
    main()

#!/usr/bin/env python
"""Fit rap_predict_latency_us's constants (RAP_MODEL_FIT in csrc/rap_plan.cpp)
to a budget sweep (scripts/budget_sweep.py JSON lines): per kernel family
T = t0 + c_work * work + c_pair * pairs + c_dense * dwork + bytes / BW, with work the busiest
CTA's predicted cost units and pairs its (sparse output, row) pairs
and dwork its serial dense cost units (rap_predict_terms); non-negative
relative least squares (a term whose fitted weight would be negative is
dropped).
usage: fit_cost_model.py SWEEP.jsonl"""
import itertools
import json
import sys

import numpy as np

BW = 6446.6  # MEASURED_PEAKS.json HBM GB/s


def fit(rows):
    y = np.array([r["measured_us"] - r["bytes"] / (BW * 1e3) for r in rows])
    if not rows:
        return 0.0, np.zeros(4)
    m = np.array([r["measured_us"] for r in rows])
    X = np.stack([np.ones(len(rows)), [r["work"] for r in rows], [r["pairs"] for r in rows],
                  [r["dwork"] for r in rows]], 1)
    best = None
    for keep in itertools.product([0, 1], repeat=3):  # non-negativity: try dropping terms
        cols = [0] + [i + 1 for i in range(3) if keep[i]]
        A = X[:, cols] / m[:, None]
        sol = np.linalg.lstsq(A, y / m, rcond=None)[0]
        if (sol < 0).any():
            continue
        k = np.zeros(4)
        k[cols] = sol
        err = (X @ k + np.array([r["bytes"] for r in rows]) / (BW * 1e3)) / m - 1
        score = float(np.sqrt(np.mean(err ** 2)))
        if best is None or score < best[0]:
            best = (score, k)
    return best


def main():
    rows = [json.loads(ln) for ln in open(sys.argv[1]) if ln.startswith("{")]
    consts = []
    for fam, name in ((1, "tiled"), (2, "rows"), (3, "generated")):
        R = [r for r in rows if r["model_kernel"] == fam]
        score, k = fit(R)
        consts += list(k)
        print(f"{name:9s} n={len(R):2d}  t0 {k[0]:7.3f} us  c_work {k[1]:.4e} us/unit  c_pair {k[2]:.4e} us/pair  "
              f"c_dense {k[3]:.4e} us/unit  rms rel err {score:.3f}")
        for r in R:
            p = k[0] + k[1] * r["work"] + k[2] * r["pairs"] + k[3] * r["dwork"] + r["bytes"] / (BW * 1e3)
            print(f"   {r['workload']:7s} b={r['budget']:3d} grid={r['grid']:4d} meas {r['measured_us']:8.1f} "
                  f"pred {p:8.1f} err {100 * (p / r['measured_us'] - 1):+4.0f}%")
    print("RAP_MODEL_FIT " + ", ".join(f"{v:.6g}" for v in consts + [BW]))


if __name__ == "__main__":
    main()

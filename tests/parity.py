"""Element-by-element comparison of the CUDA path against the oracle.

Bar (R16): lengths / offsets / values bit-exact; dense f32 within
|g - o| <= 1e-5 * |o|, or both NaN, or equal infinities (zeros exact)."""
import numpy as np

REL_TOL = 1e-5


def dense_close(g, o):
    g = np.asarray(g, dtype=np.float64)
    o = np.asarray(o, dtype=np.float64)
    both_nan = np.isnan(g) & np.isnan(o)
    eq = g == o
    rel = np.abs(g - o) <= REL_TOL * np.abs(o)
    return both_nan | eq | (np.isfinite(o) & rel)


def assert_parity(got, want, ctx=""):
    assert want["status"] == "OK", want["status"]
    for k in ("lengths", "offsets", "values"):
        a, b = np.asarray(got[k]), np.asarray(want[k])
        assert a.shape == b.shape, f"{ctx} {k}: shape {a.shape} vs {b.shape}"
        if not np.array_equal(a, b):
            bad = np.nonzero(a != b)[0]
            raise AssertionError(f"{ctx} {k}: {len(bad)} mismatches, first at {bad[:5]}: got {a[bad[:5]]} "
                                 f"want {b[bad[:5]]}")
    g, o = got["dense"], want["dense"]
    assert g.shape == o.shape, f"{ctx} dense shape {g.shape} vs {o.shape}"
    ok = dense_close(g, o)
    if not ok.all():
        r, c = np.nonzero(~ok)
        raise AssertionError(f"{ctx} dense: {len(r)} mismatches, first (row, col) {list(zip(r[:5], c[:5]))}: "
                             f"got {g[r[:5], c[:5]]} want {o[r[:5], c[:5]]}")

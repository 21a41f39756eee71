"""Small builders for hand-made test batches and graph specs (test-only)."""
import numpy as np

from paper_conf_asplos_wangwdz0d24_b200.synth import pack_bitmap


def sparse_from_lists(rows, base_offset=0, null_payload=None):
    """rows: list of list[int] | None (null).  null_payload: optional list of ids
    to place in the child segment of null rows (Arrow allows it; must be ignored)."""
    off = [base_offset]
    vals = [-99] * base_offset
    valid = []
    for r in rows:
        if r is None:
            seg = list(null_payload or [])
            valid.append(False)
        else:
            seg = list(r)
            valid.append(True)
        vals += seg
        off.append(off[-1] + len(seg))
    return (np.array(off, dtype=np.int32), np.array(vals, dtype=np.int64),
            pack_bitmap(np.array(valid, dtype=bool)))


def dense_from_values(vals):
    """vals: list of float | None (None = cleared validity bit, junk payload)."""
    x = np.array([12345.0 if v is None else v for v in vals], dtype=np.float32)
    valid = np.array([v is not None for v in vals], dtype=bool)
    return x, pack_bitmap(valid)


def batch(n_rows, dense=(), sparse=()):
    """dense: list of (x, bitmap); sparse: list of (off, vals, bitmap)."""
    return {"n_rows": n_rows,
            "dense": [d[0] for d in dense], "dense_valid": [d[1] for d in dense],
            "sp_off": [s[0] for s in sparse], "sp_val": [s[1] for s in sparse],
            "sp_valid": [s[2] for s in sparse]}


def node(op, inputs, **kw):
    d = {"op": op, "inputs": [list(x) for x in inputs]}
    d.update(kw)
    return d


def spec(n_dense, n_sparse, nodes, outputs):
    return {"n_dense": n_dense, "n_sparse": n_sparse, "nodes": nodes, "outputs": outputs}


def split_jagged(res, n_rows):
    """Per (feature, row) python lists from a result dict."""
    L, O, V = res["lengths"], res["offsets"], res["values"]
    F = len(L) // max(n_rows, 1) if n_rows else 0
    out = []
    for f in range(F):
        out.append([list(V[O[f * n_rows + b]:O[f * n_rows + b + 1]]) for b in range(n_rows)])
    return out

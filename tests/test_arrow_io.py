"""Arrow / Parquet ingestion (NEXT-2; arrow_io.py): a synthetic batch written
as an Arrow RecordBatch / a Parquet file and read back maps onto the R19 raw
layout (the same validity words, offsets and ids), and the oracle's outputs of
the read-back batch equal those of the original."""
import os

import numpy as np
import pytest

from paper_conf_asplos_wangwdz0d24_b200 import arrow_io, synth


def _valid(words, n):
    if words is None:
        return np.ones(n, dtype=bool)
    return np.unpackbits(np.asarray(words, dtype=np.uint32).view(np.uint8), bitorder="little")[:n].astype(bool)


def _same_input(a, b):
    n = a["n_rows"]
    assert b["n_rows"] == n
    for c in range(len(a["dense"])):
        va, vb = _valid(a["dense_valid"][c], n), _valid(b["dense_valid"][c], n)
        assert np.array_equal(va, vb)
        x, y = np.asarray(a["dense"][c])[va], np.asarray(b["dense"][c])[vb]
        assert np.array_equal(np.isnan(x), np.isnan(y)) and np.array_equal(x[~np.isnan(x)], y[~np.isnan(y)])
    for c in range(len(a["sp_off"])):
        va, vb = _valid(a["sp_valid"][c], n), _valid(b["sp_valid"][c], n)
        assert np.array_equal(va, vb)
        oa, ob = np.asarray(a["sp_off"][c]), np.asarray(b["sp_off"][c])
        la, lb = np.diff(oa), np.diff(ob)
        assert np.array_equal(la[va], lb[vb])
        for r in np.nonzero(va)[0][:200]:
            assert np.array_equal(np.asarray(a["sp_val"][c])[oa[r]:oa[r + 1]], np.asarray(b["sp_val"][c])[ob[r]:ob[r + 1]])


@pytest.mark.parametrize("wl,B", [("c2", 3000), ("c4", 700)])
def test_arrow_round_trip_and_oracle(wl, B):
    from oracle import oracle

    w = synth.c2_terabyte(0) if wl == "c2" else synth.c4_multihot(0, n_features=24)
    h = synth.make_batch(w, B, seed=9)
    rb = arrow_io.arrow_from_batch(h)
    back = arrow_io.batch_from_arrow(rb, [f"d{c}" for c in range(len(h["dense"]))],
                                     [f"s{c}" for c in range(len(h["sp_off"]))])
    _same_input(h, back)
    want, got = oracle.run(w.spec, h), oracle.run(w.spec, back)
    for k in ("lengths", "offsets", "values"):
        assert np.array_equal(want[k], got[k])
    assert np.array_equal(np.isnan(want["dense"]), np.isnan(got["dense"]))
    assert np.array_equal(want["dense"][~np.isnan(want["dense"])], got["dense"][~np.isnan(got["dense"])])


def test_parquet_row_groups(tmp_path):
    w = synth.c1_kaggle(0)
    bs = [synth.make_batch(w, B, seed=s) for s, B in ((1, 1024), (2, 3000), (3, 77))]
    path = os.path.join(tmp_path, "b.parquet")
    arrow_io.write_parquet(bs, path)
    back = list(arrow_io.read_parquet_batches(path, 13, 26))
    assert len(back) == 3
    for a, b in zip(bs, back):
        _same_input(a, b)


def test_arrow_views_are_zero_copy():
    """Dense data and list offsets/values of an unsliced RecordBatch are views of
    the Arrow buffers (no copy on the ingestion path)."""
    w = synth.c2_terabyte(0)
    h = synth.make_batch(w, 512, seed=4)
    rb = arrow_io.arrow_from_batch(h)
    b = arrow_io.batch_from_arrow(rb, [f"d{c}" for c in range(13)], [f"s{c}" for c in range(26)])
    assert b["dense"][0].base is not None and not b["dense"][0].flags.owndata
    assert not b["sp_off"][0].flags.owndata and not b["sp_val"][0].flags.owndata

"""Arrow / Parquet ingestion of raw batches (§6.3
L1368-1461: batches arrive as columnar data loaded by the data loader).

The raw batch layout of the C ABI (include/rap.h, R19) is Arrow's
own: a dense column is a float32 array with an LSB-first validity bitmap, a
sparse column a list<int64> array whose int32 offsets index its child values
(absolute, so a sliced array's first offset may be non-zero).  A RecordBatch
therefore maps onto the host batch without copying: `batch_from_arrow` views
the Arrow buffers as the numpy arrays `rap.DeviceBatch` (device upload) or
the host-buffer entries (`rap_preprocess_host*`) take.  Host orchestration
only -- no operator arithmetic.
"""
from __future__ import annotations

import numpy as np


def _bitmap_words(buf, n_rows: int, offset: int):
    """An Arrow validity buffer as uint32 words (bit b of word b >> 5, R19);
    None when the array has no nulls."""
    if buf is None:
        return None
    nw = (n_rows + 31) // 32
    raw = np.frombuffer(buf, dtype=np.uint8)
    if offset % 8 == 0 and len(raw) >= offset // 8 + 4 * nw:
        return raw[offset // 8: offset // 8 + 4 * nw].view(np.uint32)
    # a bit offset that is not byte aligned (a sliced array), or a short
    # buffer: repack (the only copying path)
    bits = np.unpackbits(raw, bitorder="little")[offset: offset + n_rows]
    out = np.zeros(nw * 32, dtype=np.uint8)
    out[:n_rows] = bits
    return np.packbits(out, bitorder="little").view(np.uint32)


def batch_from_arrow(rb, dense_names, sparse_names) -> dict:
    """A pyarrow RecordBatch -> the host batch dict (zero-copy views where the
    Arrow buffers already have the R19 layout).  dense_names: float32 columns,
    sparse_names: list<int64> columns, in the graph's input order."""
    import pyarrow as pa

    n = rb.num_rows
    dense, dvalid = [], []
    for name in dense_names:
        a = rb.column(name)
        if a.type != pa.float32():
            a = a.cast(pa.float32())
        bufs = a.buffers()
        data = np.frombuffer(bufs[1], dtype=np.float32)[a.offset: a.offset + n]
        dense.append(data)
        dvalid.append(_bitmap_words(bufs[0], n, a.offset) if a.null_count else None)
    soff, sval, svalid = [], [], []
    for name in sparse_names:
        a = rb.column(name)
        if not pa.types.is_list(a.type):
            raise TypeError(f"sparse column {name}: list<int64> expected, got {a.type}")
        if a.type.value_type != pa.int64():
            a = a.cast(pa.list_(pa.int64()))
        bufs = a.buffers()  # validity, offsets, child validity, child values
        off = np.frombuffer(bufs[1], dtype=np.int32)[a.offset: a.offset + n + 1]
        child = a.values
        vals = np.frombuffer(child.buffers()[1], dtype=np.int64)[child.offset: child.offset + len(child)]
        soff.append(off)
        sval.append(vals)
        svalid.append(_bitmap_words(bufs[0], n, a.offset) if a.null_count else None)
    return {"n_rows": n, "dense": dense, "dense_valid": dvalid, "sp_off": soff, "sp_val": sval, "sp_valid": svalid}


def _valid_bits(words, n):
    return np.unpackbits(words.view(np.uint8), bitorder="little")[:n].astype(bool)


def arrow_from_batch(batch: dict, dense_names=None, sparse_names=None):
    """The host batch dict -> a pyarrow RecordBatch (the synthetic data written
    as a data loader would read it)."""
    import pyarrow as pa

    n = int(batch["n_rows"])
    nd, ns = len(batch["dense"]), len(batch["sp_off"])
    dense_names = dense_names or [f"d{c}" for c in range(nd)]
    sparse_names = sparse_names or [f"s{c}" for c in range(ns)]
    cols, names = [], []
    for c in range(nd):
        v = batch["dense_valid"][c]
        mask = None if v is None else ~_valid_bits(v, n)
        cols.append(pa.array(np.asarray(batch["dense"][c], dtype=np.float32), mask=mask, type=pa.float32()))
        names.append(dense_names[c])
    for c in range(ns):
        off = np.asarray(batch["sp_off"][c], dtype=np.int32)
        vals = np.asarray(batch["sp_val"][c], dtype=np.int64)
        v = batch["sp_valid"][c]
        # absolute offsets into the child: rebase onto a child that starts at off[0]
        child = pa.array(vals[off[0]: off[-1]], type=pa.int64())
        rel = pa.array(off - off[0], type=pa.int32())
        mask = None if v is None else pa.array(~_valid_bits(v, n))
        cols.append(pa.ListArray.from_arrays(rel, child, mask=mask))
        names.append(sparse_names[c])
    return pa.RecordBatch.from_arrays(cols, names=names)


def write_parquet(batches, path: str):
    """Host batch dicts -> one Parquet file (one row group per batch)."""
    import pyarrow as pa
    import pyarrow.parquet as pq

    rbs = [arrow_from_batch(b) for b in batches]
    with pq.ParquetWriter(path, rbs[0].schema) as wr:  # each batch its own row group
        for rb in rbs:
            wr.write_table(pa.Table.from_batches([rb]), row_group_size=rb.num_rows)


def read_parquet_batches(path: str, n_dense: int, n_sparse: int):
    """Yield the host batch dict of every row group of a Parquet file written
    by write_parquet (column names d<c>, s<c>)."""
    import pyarrow.parquet as pq

    f = pq.ParquetFile(path)
    dn, sn = [f"d{c}" for c in range(n_dense)], [f"s{c}" for c in range(n_sparse)]
    for g in range(f.num_row_groups):
        t = f.read_row_group(g).combine_chunks()
        for rb in t.to_batches():
            yield batch_from_arrow(rb, dn, sn)

"""Arrow / Parquet ingestion end to end on the GPU (NEXT-2): a batch read back
from a Parquet file (arrow_io) preprocessed through the device entry and
through the pipelined host-buffer entry (two plans, two streams) equals the
oracle's outputs of the original batch."""
import os

import numpy as np
import pytest

from tests.parity import assert_parity

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def env():
    import torch

    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from oracle import oracle
    from paper_conf_asplos_wangwdz0d24_b200 import arrow_io, rap, synth

    rap.load()
    return rap, synth, oracle, torch, arrow_io


def test_parquet_batches_device_and_host_pipeline(env, tmp_path):
    rap, synth, oracle, torch, arrow_io = env
    w = synth.c2_terabyte(0)
    bs = [synth.make_batch(w, B, seed=20 + B) for B in (3000, 4099)]
    path = os.path.join(tmp_path, "c2.parquet")
    arrow_io.write_parquet(bs, path)
    back = list(arrow_io.read_parquet_batches(path, 13, 26))
    plans = [rap.Plan(w.spec, device=0), rap.Plan(w.spec, device=0)]
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    outs = []
    for i, (orig, b) in enumerate(zip(bs, back)):
        want = oracle.run(w.spec, orig)
        raw = rap.DeviceBatch(b, "cuda:0")
        out = rap.DeviceOutput(plans[0], b["n_rows"], raw.sp_nnz, "cuda:0")
        plans[0].preprocess(raw, out)
        torch.cuda.synchronize()
        assert_parity(out.to_numpy(), want)
        hraw = rap.DeviceBatch(b, None, pin=True)
        hout = rap.DeviceOutput(plans[i % 2], b["n_rows"], hraw.sp_nnz, None, pin=True)
        plans[i % 2].preprocess_host_async(hraw, hout, streams[i % 2])
        outs.append((hraw, hout, want))
    torch.cuda.synchronize()
    for _, hout, want in outs:
        assert_parity(hout.to_numpy(), want)
    for p in plans:
        p.close()

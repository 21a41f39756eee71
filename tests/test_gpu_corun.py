"""Layer-aligned co-run scheduling (§7.1 Algorithm 1; corun.py):
the chunked, layer-triggered launches chain into one KJT equal to the
oracle's, Algorithm 1's greedy respects the layers' order, and a co-run step
with the chunks completes."""
import numpy as np
import pytest

from tests.parity import assert_parity

pytestmark = pytest.mark.gpu


def test_layer_aligned_chunks_equal_oracle():
    import torch

    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from oracle import oracle
    from paper_conf_asplos_wangwdz0d24_b200 import corun, rap, synth

    w = synth.c2_terabyte(0)
    B = 3000
    h = synth.make_batch(w, B, seed=61)
    raw = rap.DeviceBatch(h, "cuda:0")
    # windows small enough that the 34 outputs spread over several layers
    layer_us = {n: 6.0 for n in corun.DLRMStep.LAYERS}
    lap = corun.LayerAlignedPrep(w.spec, B, raw.sp_nnz, layer_us, device=0)
    assert len(lap.chunks) > 1
    order = [c["layer"] for c in lap.chunks]
    assert order == [n for n in corun.DLRMStep.LAYERS if n in order]  # step order, each layer once
    assert sum(len(c["outputs"]) for c in lap.chunks) == 34
    assert all(1 <= c["budget"] <= 148 for c in lap.chunks)
    out = lap.output(raw.sp_nnz, "cuda:0")
    s = torch.cuda.Stream()
    for layer in corun.DLRMStep.LAYERS:  # in layer order, as a step would
        lap.launch(raw, out, s, layer)
    s.synchronize()
    got = out.to_numpy()
    got.pop("features")
    assert_parity(got, oracle.run(w.spec, h), "layer-aligned chunks")
    # one co-run step with a small training step
    train = corun.DLRMStep("cuda:0", batch=1024, table_rows=[1000] * 26)
    t, p, a = corun.measure_layer_aligned(lap, [raw], [out], train, steps=4, warmup=1)
    assert t > 0 and p > 0 and a > 0
    lap.close()

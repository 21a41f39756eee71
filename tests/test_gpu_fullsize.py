"""Parity of the launches bench.py times, at their full size, against the
oracle (VERDICT r01 "parity holes"): config 4 (512 multi-hot features,
FillNull -> Clamp -> SigridHash -> FirstX(32)) at the bench's batch and seed,
compared completely, in the default kernel selection the bench uses (AUTO).
C2 at 65536 rows is compared completely in tests/test_gpu_parity.py.
Integer outputs bit-exact (tests/parity.py)."""
import numpy as np
import pytest

from tests.parity import assert_parity

pytestmark = pytest.mark.gpu

C4_BATCH = 16384  # bench.py --c4-batch default
C4_SEEDS = (700, 701)  # bench.py c4_point's two rotating batches


@pytest.fixture(scope="module")
def env():
    import torch

    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from oracle import oracle
    from paper_conf_asplos_wangwdz0d24_b200 import rap, synth

    rap.load()
    return rap, synth, oracle, torch


def test_c4_bench_launch_full(env):
    rap, synth, oracle, torch = env
    w = synth.c4_multihot(0)
    plan = rap.Plan(w.spec, device=0)
    h = synth.make_batch(w, C4_BATCH, seed=C4_SEEDS[0])
    raw = rap.DeviceBatch(h, "cuda:0")
    out = rap.DeviceOutput(plan, C4_BATCH, raw.sp_nnz, "cuda:0")
    plan.preprocess(raw, out)
    torch.cuda.synchronize()
    assert plan.check_overflow() == 0
    got = out.to_numpy()
    info = plan.info()
    plan.close()
    del raw, out
    torch.cuda.empty_cache()
    want = oracle.run(w.spec, h)
    assert_parity(got, want, ctx=f"c4 B={C4_BATCH} kernel {info['kernel_last']}")
    # the launch moves ~1.3e8 ids: FirstX(32) of Poisson(20*w_f) lists
    assert got["values"].shape[0] > 100 * C4_BATCH * 512 // 10


def test_c4_second_batch_rows_sampled(env):
    """The bench's second rotating batch through the same plan (cached
    partition for a new shape): rows sampled at tiles' edges and the tail."""
    rap, synth, oracle, torch = env
    from tests.test_dist import _slice_batch

    w = synth.c4_multihot(0)
    plan = rap.Plan(w.spec, device=0)
    outs = []
    for seed in C4_SEEDS:
        h = synth.make_batch(w, C4_BATCH, seed=seed)
        raw = rap.DeviceBatch(h, "cuda:0")
        out = rap.DeviceOutput(plan, C4_BATCH, raw.sp_nnz, "cuda:0")
        plan.preprocess(raw, out)
        outs.append((h, raw, out))
    torch.cuda.synchronize()
    h, _, out = outs[1]
    B, F = C4_BATCH, 512
    L = out.lengths.cpu().numpy().reshape(-1)
    O = out.offsets.cpu().numpy()
    assert O[0] == 0 and np.array_equal(np.diff(O), L)
    V = out.values
    for r0, n in ((0, 160), (4064, 96), (8192, 64), (B - 224, 224)):
        want = oracle.run(w.spec, _slice_batch(h, r0, n))
        assert want["status"] == "OK"
        Lw, Ow, Vw = want["lengths"].reshape(F, n), want["offsets"], want["values"]
        assert np.array_equal(L.reshape(F, B)[:, r0:r0 + n], Lw), r0
        for f in range(F):
            a, b = O[f * B + r0], O[f * B + r0 + n]
            assert np.array_equal(V[a:b].cpu().numpy(), Vw[Ow[f * n]:Ow[f * n + n]]), (r0, f)
    plan.close()

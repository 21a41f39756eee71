"""Cast (Table 1; reading R13): the jagged values emitted as
int32 (RAP_OUT_VALUES_I32).  Every case runs on the three fused kernels and
compares element by element with the oracle's int64 ids cast by two's
complement ((int32_t)id, numpy astype; pinned in test_oracle_pins.py)."""
import numpy as np
import pytest

from tests.helpers import batch, node, sparse_from_lists, spec
from tests.parity import assert_parity

pytestmark = pytest.mark.gpu

I64_MIN, I64_MAX = -(2**63), 2**63 - 1


@pytest.fixture(scope="module")
def env():
    import torch

    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from oracle import oracle
    from paper_conf_asplos_wangwdz0d24_b200 import rap, synth

    rap.load()
    return rap, synth, oracle, torch


@pytest.fixture(params=[1, 2, 3], ids=["tiled", "rows", "jit"])
def kmode(request):
    return request.param


def run_cast(env, kmode, spec_, host):
    rap, _, oracle, torch = env
    want = oracle.run(spec_, host)
    assert want["status"] == "OK"
    plan = rap.Plan(spec_, device=0)
    plan.set_kernel(kmode)
    raw = rap.DeviceBatch(host, "cuda:0")
    out = rap.DeviceOutput(plan, host["n_rows"], raw.sp_nnz, "cuda:0", values_i32=True)
    plan.preprocess(raw, out)
    torch.cuda.synchronize()
    got = out.to_numpy()
    plan.close()
    assert got["values"].dtype == np.int32
    want = dict(want)
    want["values"] = np.asarray(want["values"], dtype=np.int64).astype(np.int32)
    assert_parity(got, want)


@pytest.mark.parametrize("wl,B", [("c1", 4096), ("c2", 3000), ("c2", 65536), ("c4", 1500), ("plan2", 2000)])
def test_cast_int32_configs(env, kmode, wl, B):
    _, synth, _, _ = env
    if wl == "c4" and kmode != 1:
        pytest.skip("512 raw columns: the tiled kernel only (rap_set_kernel rows / jit: UNSUPPORTED)")
    w = {"c1": synth.c1_kaggle, "c2": synth.c2_terabyte, "c4": synth.c4_multihot,
         "plan2": lambda s: synth.plan_graph(2, s)}[wl](0)
    run_cast(env, kmode, w.spec, synth.make_batch(w, B, seed=B + 3))


def test_cast_int32_wraps_large_ids(env, kmode):
    """Ids beyond 2^31 (SigridHash with M = 2^40, raw ids at the int64
    extremes through FirstX): the cast keeps the low 32 bits."""
    rng = np.random.default_rng(4)
    B = 1200
    rows = [list(rng.integers(-(2**40), 2**40, size=int(rng.integers(0, 4)))) for _ in range(B)]
    rows[3] = [I64_MIN, I64_MAX, 2**31, 2**32 + 7]
    sp = sparse_from_lists(rows)
    nodes = [node("sigridhash", [("s", 0)], salt=9, max_value=2**40),
             node("firstx", [("s", 0)], x=3)]
    run_cast(env, kmode, spec(0, 1, nodes, [0, 1]), batch(B, sparse=[sp]))


def test_cast_rejected_on_host_entries_and_chains(env):
    rap, synth, _, torch = env
    w = synth.c1_kaggle(0)
    host = synth.make_batch(w, 256, seed=1)
    plan = rap.Plan(w.spec, device=0)
    hraw = rap.DeviceBatch(host, None, pin=True)
    hout = rap.DeviceOutput(plan, 256, hraw.sp_nnz, None, pin=True, values_i32=True)
    with pytest.raises(rap.RapError):
        plan.preprocess_host(hraw, hout)
    raw = rap.DeviceBatch(host, "cuda:0")
    out = rap.DeviceOutput(plan, 256, raw.sp_nnz, "cuda:0", values_i32=True)
    out.struct.flags |= rap.OUT_CHAIN
    with pytest.raises(rap.RapError):
        plan.preprocess(raw, out)
    plan.close()

"""The co-running cost model (rap_predict_latency_us; PAPER.md
§5.2) against kernel times measured here: within +-25% for
configs 1, 2 and 4 at budgets 16 / 37 / 74 / 148 (+-30% for config 1 at <= 37
SMs, where the generated kernel's per-warp chain dominates; VERDICT r01 item
6); the
model replays the launch the plan makes (kernel and grid equal the plan's
own); rap_choose_budget picks the smallest budget whose prediction fits the
overlap capacity (T_delta = P - OC <= 0, L1138-1152)."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

BUDGETS = (16, 37, 74, 148)


@pytest.fixture(scope="module")
def env():
    import torch

    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_asplos_wangwdz0d24_b200 import rap, synth

    rap.load()
    return rap, synth, torch


def _time(torch, plan, sets, steps):
    s = torch.cuda.current_stream()
    for i in range(4):
        plan.preprocess(*sets[i % len(sets)], s)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for i in range(steps):
        plan.preprocess(*sets[i % len(sets)], s)
    e1.record(s)
    e1.synchronize()
    return e0.elapsed_time(e1) / steps * 1e3


@pytest.mark.parametrize("wl,B", [("c1", 4096), ("c2", 65536), ("c4", 16384)])
def test_predicted_latency_within_25_percent(env, wl, B):
    rap, synth, torch = env
    w = {"c1": synth.c1_kaggle, "c2": synth.c2_terabyte, "c4": synth.c4_multihot}[wl](0)
    plan = rap.Plan(w.spec, device=0)
    sets = []
    for i in range(2 if wl == "c4" else 3):
        r = rap.DeviceBatch(synth.make_batch(w, B, seed=950 + i), "cuda:0")
        sets.append((r, rap.DeviceOutput(plan, B, r.sp_nnz, "cuda:0")))
    nnz = sets[0][0].sp_nnz
    errs = []
    for b in BUDGETS:
        plan.set_budget(b)
        meas = _time(torch, plan, sets, 10 if wl == "c4" else 40)
        pred = plan.predict_latency_us(B, nnz, b)
        fam, grid = plan.predict_terms(B, nnz, b)[:2]
        info = plan.info()
        assert (fam, grid) == (info["kernel_last"], info["grid"]), (b, fam, grid, info["kernel_last"], info["grid"])
        errs.append((b, round(meas, 1), round(pred, 1)))
        # generated kernel at small grids: the serial per-output chain of a warp
        # (op-mix dependent) is only approximated by the pairs term -- the fit's
        # worst case is C1 at 16 SMs, -26% (profiles/r02b_cost_model_fit.txt)
        tol = 0.30 if (wl == "c1" and b <= 37) else 0.25
        assert abs(pred / meas - 1) <= tol, errs
    plan.close()


def test_choose_budget_fits_overlap_capacity(env):
    rap, synth, torch = env
    w = synth.c2_terabyte(0)
    B = 65536
    plan = rap.Plan(w.spec, device=0)
    nnz = rap.DeviceBatch(synth.make_batch(w, 512, seed=1), None, pin=True).sp_nnz * (B // 512)
    preds = [plan.predict_latency_us(B, nnz, b) for b in range(1, 149)]
    for oc in (60.0, 150.0, 600.0, 5000.0):
        b, td = plan.choose_budget(B, nnz, oc)
        assert td == pytest.approx(preds[b - 1] - oc)
        if td <= 0:  # smallest budget that fits
            assert all(p > oc for p in preds[: b - 1])
        else:  # none fits: the best (smallest T_delta)
            assert td == pytest.approx(min(preds) - oc)
    b_small, _ = plan.choose_budget(B, nnz, 5000.0)
    b_large, _ = plan.choose_budget(B, nnz, 150.0)
    assert b_small < b_large
    plan.close()

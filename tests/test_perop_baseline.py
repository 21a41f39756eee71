"""The sequential per-op baseline (baselines/perop_torch.py, bench.py's
"perop" arm: one eager PyTorch evaluation per graph node) computes the same
outputs as the oracle, so the fused kernel's speedup over it compares equal
work.  CPU here; the same code on cuda:0 in the gpu-marked case."""
import pytest

from tests.parity import assert_parity


def _check(device, w, B, seed):
    from baselines.perop_torch import PerOpGraph
    from oracle import oracle
    from paper_conf_asplos_wangwdz0d24_b200 import synth

    h = synth.make_batch(w, B, seed=seed)
    g = PerOpGraph(w.spec, device)
    got = {k: v.cpu().numpy() for k, v in g.run(g.upload(h)).items()}
    assert_parity(got, oracle.run(w.spec, h), w.name)


@pytest.mark.parametrize("wl", ["c1", "c2", "plan2"])
def test_perop_baseline_matches_oracle_cpu(wl):
    from paper_conf_asplos_wangwdz0d24_b200 import synth

    w = {"c1": synth.c1_kaggle, "c2": synth.c2_terabyte, "plan2": lambda s: synth.plan_graph(2, s)}[wl](0)
    _check("cpu", w, 1333, 5)


@pytest.mark.gpu
def test_perop_baseline_matches_oracle_gpu():
    import torch

    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_asplos_wangwdz0d24_b200 import synth

    _check("cuda:0", synth.c2_terabyte(0), 4000, 6)

"""SM partition streams (rap_sm_partition_stream, a CUDA green context):
the fused kernels run on a hardware partition of the SMs and produce the
oracle's outputs (§6.2)."""
import pytest

from tests.parity import assert_parity

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("kmode", [1, 3])
def test_partition_stream_parity(kmode):
    import torch

    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from oracle import oracle
    from paper_conf_asplos_wangwdz0d24_b200 import rap, synth

    part = rap.SMPartitionStream(0, 16)
    assert part.sms >= 16 and part.sms % 8 == 0 and part.sms < 148
    w = synth.c2_terabyte(0)
    h = synth.make_batch(w, 5000, seed=71)
    plan = rap.Plan(w.spec, device=0, sm_budget=part.sms)
    plan.set_kernel(kmode)
    raw = rap.DeviceBatch(h, "cuda:0")
    out = rap.DeviceOutput(plan, 5000, raw.sp_nnz, "cuda:0")
    for _ in range(2):
        plan.preprocess(raw, out, part.stream)
    part.stream.synchronize()
    assert_parity(out.to_numpy(), oracle.run(w.spec, h), f"partition kernel {kmode}")
    plan.close()
    part.close()

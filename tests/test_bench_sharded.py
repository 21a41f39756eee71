"""bench.py's N > 1 path (run_sharded) end to end on one GPU: two ranks under
torch.distributed.run with the gloo backend (host-staged residual exchange;
NCCL cannot run two ranks on one device).  Checks the JSON line's contract
keys, the skewed placement's residual move and the config-4 per-N point."""
import json
import os
import socket
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.gpu
def test_bench_two_ranks_gloo_one_gpu():
    import torch

    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
           "127.0.0.1", "--master-port", str(port), "bench.py", "--gpus", "2", "--dist-backend", "gloo",
           "--steps", "3", "--warmup", "3", "--batch", "8192", "--c4-batch", "2048", "--placement", "skewed",
           "--imbalance-tol", "0.05"]
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["steps"] == 3 and d["warmup"] == 3 and d["scaling"] == "strong"
    assert d["value"] > 0 and d["config"]["batch"] == 8192
    assert d["config"]["comm_model"]["us_per_unit"] > 0
    assert d["config"]["rank0_sparse_columns"] <= 26
    assert d["c4"]["value"] > 0 and 0 < d["c4"]["tables_per_rank"] < 512

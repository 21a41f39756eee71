#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
TAG=denselate timeout 120 python scripts/cold_trace.py
RAP_JIT_DENSE_LATE=0 STAMPS=0 TAG=dense-early timeout 120 python scripts/cold_trace.py
) > gpurun_out/r4g.log 2>&1
grep -E "graph|^c|span|->|kernel end|staged|totals|dense warp" gpurun_out/r4g.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -m gpu -k "jit" > gpurun_out/r4g_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r4g_pytest.log
tail -2 gpurun_out/r4g_pytest.log

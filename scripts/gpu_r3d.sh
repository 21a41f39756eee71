#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 300 python scripts/cold_trace.py > gpurun_out/r3d_trace.log 2>&1
RAP_JIT_IDS=0 STAMPS=0 TAG=noids timeout 300 python scripts/cold_trace.py >> gpurun_out/r3d_trace.log 2>&1
cat gpurun_out/r3d_trace.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_fullsize.py -q -x -m gpu -k "jit or fullsize or full" > gpurun_out/r3d_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r3d_pytest.log
tail -5 gpurun_out/r3d_pytest.log

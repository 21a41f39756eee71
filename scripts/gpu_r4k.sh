#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
TAG=tail20 timeout 120 python scripts/cold_trace.py
RAP_JIT_TAIL_PCT=0 STAMPS=0 TAG=tail0 timeout 120 python scripts/cold_trace.py
RAP_JIT_TAIL_PCT=12 STAMPS=0 TAG=tail12 timeout 120 python scripts/cold_trace.py
RAP_JIT_TAIL_PCT=30 STAMPS=0 TAG=tail30 timeout 120 python scripts/cold_trace.py
) > gpurun_out/r4k.log 2>&1
grep -E "graph|^c|span|->|kernel end|dense warp" gpurun_out/r4k.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_fullsize.py tests/test_gpu_cast.py -q -x -m gpu -k "jit" > gpurun_out/r4k_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r4k_pytest.log
tail -2 gpurun_out/r4k_pytest.log; grep -E "^FAILED|Error" gpurun_out/r4k_pytest.log | head -5

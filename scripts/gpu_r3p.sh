#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
STAMPS=0 TAG=tabs timeout 300 python scripts/cold_trace.py
RAP_JIT_TABS=0 STAMPS=0 TAG=notabs timeout 300 python scripts/cold_trace.py
RAP_JIT_TAB_BYTES=8192 STAMPS=0 TAG=samples-only timeout 300 python scripts/cold_trace.py
RAP_JIT_SMALL_B=1 WL=c1 B=4096 STAMPS=0 TAG=c1jit-tabs timeout 300 python scripts/cold_trace.py
) > gpurun_out/r3p.log 2>&1
grep -E "graph|^c" gpurun_out/r3p.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_fullsize.py -q -x -m gpu -k "jit or fullsize or full" > gpurun_out/r3p_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r3p_pytest.log
tail -3 gpurun_out/r3p_pytest.log; grep -E "^FAILED|Error" gpurun_out/r3p_pytest.log | head -5

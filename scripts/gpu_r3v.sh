#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
TAG=loop timeout 300 python scripts/cold_trace.py
RAP_JIT_LOOP=0 STAMPS=0 TAG=batched timeout 300 python scripts/cold_trace.py
RAP_JIT_SMALL_B=1 WL=c1 B=4096 STAMPS=0 TAG=c1jit-loop timeout 300 python scripts/cold_trace.py
) > gpurun_out/r3v.log 2>&1
grep -E "graph|^c|span|->|kernel end|staged|totals" gpurun_out/r3v.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_fullsize.py -q -x -m gpu -k "jit or fullsize or full" > gpurun_out/r3v_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r3v_pytest.log
tail -3 gpurun_out/r3v_pytest.log; grep -E "^FAILED|Error" gpurun_out/r3v_pytest.log | head -5

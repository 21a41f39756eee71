#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
RAP_JIT_PDL=1 STAMPS=0 TAG=pdl timeout 120 python scripts/cold_trace.py
STAMPS=0 TAG=nopdl timeout 120 python scripts/cold_trace.py
) > gpurun_out/r4i.log 2>&1
cat gpurun_out/r4i.log | grep -E "graph|^c|Error|error" | head
RAP_JIT_PDL=1 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -m gpu -k "jit" > gpurun_out/r4i_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r4i_pytest.log
tail -2 gpurun_out/r4i_pytest.log; grep -E "^FAILED|Error" gpurun_out/r4i_pytest.log | head -5

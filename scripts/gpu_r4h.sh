#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
TAG=basesdense timeout 120 python scripts/cold_trace.py
RAP_JIT_BASES_DENSE=0 STAMPS=0 TAG=bases-sparse timeout 120 python scripts/cold_trace.py
) > gpurun_out/r4h.log 2>&1
grep -E "graph|^c|span|->|kernel end|staged|totals|dense warp" gpurun_out/r4h.log
timeout 1800 python -m pytest tests -q -x -m gpu > gpurun_out/r4h_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r4h_pytest.log
tail -2 gpurun_out/r4h_pytest.log; grep -E "^FAILED|Error" gpurun_out/r4h_pytest.log | head -5

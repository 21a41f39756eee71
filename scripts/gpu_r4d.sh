#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
STAMPS=0 TAG=blkcap timeout 120 python scripts/cold_trace.py
) > gpurun_out/r4d.log 2>&1
grep -E "graph|^c" gpurun_out/r4d.log
timeout 1800 python -m pytest tests -q -x -m gpu > gpurun_out/r4d_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r4d_pytest.log
tail -2 gpurun_out/r4d_pytest.log; grep -E "^FAILED|Error" gpurun_out/r4d_pytest.log | head -5

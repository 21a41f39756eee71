#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
TAG=suptotals timeout 300 python scripts/cold_trace.py
KMODE=2 STAMPS=0 TAG=interp timeout 300 python scripts/cold_trace.py
) > gpurun_out/r3z.log 2>&1
grep -E "graph|^c|span|->|kernel end|staged|totals|dense warp" gpurun_out/r3z.log
timeout 1800 python -m pytest tests -q -x -m gpu > gpurun_out/r3z_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r3z_pytest.log
tail -2 gpurun_out/r3z_pytest.log; grep -E "^FAILED|Error" gpurun_out/r3z_pytest.log | head -5

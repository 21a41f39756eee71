#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
timeout 300 python scripts/cold_trace.py
) > gpurun_out/r3c.log 2>&1
cat gpurun_out/r3c.log

#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
RAP_JIT_SKIP=15 RAP_JIT_NOSTORE=1 TAG=skip15nostore timeout 300 python scripts/cold_trace.py
RAP_JIT_SKIP=16 TAG=emptyemit timeout 300 python scripts/cold_trace.py
RAP_JIT_SKIP=15 TAG=skip15 timeout 300 python scripts/cold_trace.py
) > gpurun_out/r3j.log 2>&1
grep -E "graph|^c2|span|->|kernel end|dense warp|staged|totals" gpurun_out/r3j.log

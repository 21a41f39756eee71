#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
STAMPS=0 TAG=dw3-t20 timeout 120 python scripts/cold_trace.py
RAP_JIT_DENSE_WARPS=4 STAMPS=0 TAG=dw4-t20 timeout 120 python scripts/cold_trace.py
RAP_JIT_DENSE_WARPS=4 RAP_JIT_TAIL_PCT=28 STAMPS=0 TAG=dw4-t28 timeout 120 python scripts/cold_trace.py
RAP_JIT_DENSE_WARPS=2 RAP_JIT_TAIL_PCT=12 STAMPS=0 TAG=dw2-t12 timeout 120 python scripts/cold_trace.py
) > gpurun_out/r4m.log 2>&1
grep -E "graph|^c" gpurun_out/r4m.log

#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
STAMPS=0 TAG=base timeout 300 python scripts/cold_trace.py
RAP_JIT_MINB=3 RAP_RB_ROWS=224 STAMPS=0 TAG=minb3rows224 timeout 300 python scripts/cold_trace.py
RAP_JIT_MINB=4 RAP_RB_ROWS=224 STAMPS=0 TAG=minb4rows224 timeout 300 python scripts/cold_trace.py
RAP_JIT_MINB=4 STAMPS=0 TAG=minb4 timeout 300 python scripts/cold_trace.py
RAP_JIT_MINB=3 STAMPS=0 TAG=minb3 timeout 300 python scripts/cold_trace.py
) > gpurun_out/r3l.log 2>&1
grep -E "graph|^c" gpurun_out/r3l.log

#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
TAG=batch8 STAMPS=0 timeout 300 python scripts/cold_trace.py
RAP_JIT_SKIP=1 STAMPS=0 TAG=batch8-nomap timeout 300 python scripts/cold_trace.py
RAP_JIT_SKIP=1 RAP_JIT_BATCH=0 STAMPS=0 TAG=nobatch-nomap timeout 300 python scripts/cold_trace.py
RAP_JIT_SKIP=9 STAMPS=0 TAG=batch8-nomap-nongram timeout 300 python scripts/cold_trace.py
RAP_JIT_SKIP=9 RAP_JIT_BATCH=0 STAMPS=0 TAG=nobatch-nomap-nongram timeout 300 python scripts/cold_trace.py
) > gpurun_out/r3t.log 2>&1
grep -E "graph|^c" gpurun_out/r3t.log

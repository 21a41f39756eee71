#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
STAMPS=0 TAG=default timeout 300 python scripts/cold_trace.py
RAP_JIT_STCS=1 STAMPS=0 TAG=stcs timeout 300 python scripts/cold_trace.py
RAP_JIT_NOSTORE=1 STAMPS=0 TAG=nostore1 timeout 300 python scripts/cold_trace.py
WL=c1 B=4096 STAMPS=0 TAG=c1 timeout 300 python scripts/cold_trace.py
) > gpurun_out/r3f.log 2>&1
cat gpurun_out/r3f.log

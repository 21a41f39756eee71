#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
STAMPS=0 TAG=stcs timeout 300 python scripts/cold_trace.py
RAP_JIT_LDCS=1 STAMPS=0 TAG=stcs+ldcs timeout 300 python scripts/cold_trace.py
KMODE=2 STAMPS=0 TAG=interp-stcs timeout 300 python scripts/cold_trace.py
WL=c1 B=4096 STAMPS=0 TAG=c1 timeout 300 python scripts/cold_trace.py
WL=c1 B=4096 KMODE=3 STAMPS=0 TAG=c1jit timeout 300 python scripts/cold_trace.py
WL=c4 B=16384 NSETS=2 STAMPS=0 TAG=c4 timeout 300 python scripts/cold_trace.py
) > gpurun_out/r3g.log 2>&1
cat gpurun_out/r3g.log

#!/bin/bash
# warm vs cold phase stamps of the generated C2 kernel (+ knobs)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
timeout 300 python scripts/cold_trace.py
RAP_JIT_AHEAD=12 TAG=ahead12 STAMPS=0 timeout 300 python scripts/cold_trace.py
NSETS=2 TAG=nsets2 STAMPS=0 timeout 300 python scripts/cold_trace.py
KMODE=2 TAG=interp STAMPS=0 timeout 300 python scripts/cold_trace.py
WL=c1 B=4096 timeout 300 python scripts/cold_trace.py
) > gpurun_out/r3a.log 2>&1
cat gpurun_out/r3a.log

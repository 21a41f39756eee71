#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
STAMPS=0 TAG=map2 timeout 300 python scripts/cold_trace.py
RAP_JIT_MAP1=1 STAMPS=0 TAG=map1 timeout 300 python scripts/cold_trace.py
RAP_JIT_STPLAIN=1 STAMPS=0 TAG=map2+stplain timeout 300 python scripts/cold_trace.py
RAP_JIT_PAIRS=1 STAMPS=0 TAG=pairs+map2 timeout 300 python scripts/cold_trace.py
RAP_JIT_PAIRS=1 RAP_JIT_STPLAIN=1 STAMPS=0 TAG=pairs+map2+stplain timeout 300 python scripts/cold_trace.py
RAP_JIT_SMALL_B=1 WL=c1 B=4096 STAMPS=0 TAG=c1jit timeout 300 python scripts/cold_trace.py
RAP_JIT_SMALL_B=1 RAP_JIT_STPLAIN=1 WL=c1 B=4096 STAMPS=0 TAG=c1jit+stplain timeout 300 python scripts/cold_trace.py
) > gpurun_out/r3o.log 2>&1
grep -E "graph|^c" gpurun_out/r3o.log

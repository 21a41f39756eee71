#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
STAMPS=0 TAG=batch8 timeout 300 python scripts/cold_trace.py
RAP_JIT_BATCHSYNC=1 STAMPS=0 TAG=batch8sync timeout 300 python scripts/cold_trace.py
RAP_JIT_BATCHSYNC=1 RAP_JIT_BATCH=4 STAMPS=0 TAG=batch4sync timeout 300 python scripts/cold_trace.py
RAP_JIT_BATCHSYNC=1 RAP_JIT_BATCH=2 STAMPS=0 TAG=batch2sync timeout 300 python scripts/cold_trace.py
) > gpurun_out/r3u.log 2>&1
grep -E "graph|^c" gpurun_out/r3u.log

#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
STAMPS=0 TAG=base timeout 300 python scripts/cold_trace.py
for n in 1 2 4 8 15; do RAP_JIT_SKIP=$n STAMPS=0 TAG=skip$n timeout 300 python scripts/cold_trace.py; done
RAP_JIT_SKIP=15 RAP_JIT_NOSTORE=1 STAMPS=0 TAG=skip15nostore timeout 300 python scripts/cold_trace.py
) > gpurun_out/r3h.log 2>&1
grep -E "graph|^c2" gpurun_out/r3h.log

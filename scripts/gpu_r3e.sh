#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
STAMPS=0 TAG=default timeout 300 python scripts/cold_trace.py
for n in 1 2 3; do RAP_JIT_NOSTORE=$n STAMPS=0 TAG=nostore$n timeout 300 python scripts/cold_trace.py; done
RAP_JIT_NOSTORE=1 TAG=nostore1 timeout 300 python scripts/cold_trace.py | grep -E "bases->ids|span"
) > gpurun_out/r3e.log 2>&1
cat gpurun_out/r3e.log

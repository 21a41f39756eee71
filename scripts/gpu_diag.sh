#!/bin/bash
# Phase traces of C2 slices + ncu --set full of two slices (dev tool).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for k in ${TRACE_KEEPS:-15:16 41:42 15:41 0:49}; do KEEP=$k timeout 300 python scripts/trace.py 2>&1 | tail -6; done
KEEPS="${NCU_KEEPS:-15:16 41:42 0:49}" bash scripts/ncu_sub.sh > /dev/null 2>&1
ls gpurun_out

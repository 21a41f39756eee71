#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
WL=c4 B=16384 NSETS=2 STAMPS=0 TAG=c4-min3 timeout 300 python scripts/cold_trace.py
RAP_NVCC_FLAGS=-DRAP_MIN_CTAS=2 python -c "from paper_conf_asplos_wangwdz0d24_b200 import _build; _build.build(force=True)"
WL=c4 B=16384 NSETS=2 STAMPS=0 TAG=c4-min2 timeout 300 python scripts/cold_trace.py
RAP_NVCC_FLAGS=-DRAP_MIN_CTAS=4 python -c "from paper_conf_asplos_wangwdz0d24_b200 import _build; _build.build(force=True)"
WL=c4 B=16384 NSETS=2 STAMPS=0 TAG=c4-min4 timeout 300 python scripts/cold_trace.py
) > gpurun_out/r4c.log 2>&1
grep -E "graph|^c" gpurun_out/r4c.log

#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
KMODE=3 WL=c2 B=65536 timeout 120 python scripts/trace_rows.py 2>&1 | tail -12
KMODE=2 WL=c2 B=65536 timeout 120 python scripts/trace_rows.py 2>&1 | tail -12

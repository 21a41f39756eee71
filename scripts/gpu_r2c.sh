#!/bin/bash
# round 2, call C: row-block kernel phase trace + ncu capture
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
WL=c1 B=32 timeout 120 python scripts/trace_rows.py 2>&1 | tail -9
WL=c1 B=4096 timeout 120 python scripts/trace_rows.py 2>&1 | tail -9
WL=c2 B=65536 timeout 120 python scripts/trace_rows.py 2>&1 | tail -9
RAP_KERNEL=2 timeout 600 ncu --set full --clock-control none --import-source on -k regex:rap_rows -s 5 -c 1 -o gpurun_out/r02c_rows_c2 -f python bench.py --profile --steps 8 --warmup 5 > gpurun_out/r02c_ncu.log 2>&1
tail -3 gpurun_out/r02c_ncu.log

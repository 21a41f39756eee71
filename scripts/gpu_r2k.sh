#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
KMODE=3 WL=c2 B=65536 timeout 120 python scripts/trace_rows.py 2>&1 | tail -13
RAP_KERNEL=3 WL=c2 SIZES=65536 timeout 300 python scripts/fixed_cost.py 2>&1 | grep -v "^{"
RAP_KERNEL=3 timeout 600 ncu --set full --clock-control none --import-source on -k regex:rap_jit -s 5 -c 1 -o gpurun_out/r02k_jit_c2 -f python bench.py --profile --steps 8 --warmup 5 > gpurun_out/r02k_ncu.log 2>&1
tail -1 gpurun_out/r02k_ncu.log

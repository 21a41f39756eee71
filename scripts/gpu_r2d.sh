#!/bin/bash
# round 2, call D: row-block kernel v2 — parity, trace, fixed cost, bench, ncu
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "rows" -x > gpurun_out/r02d_pytest_rows.log 2>&1; echo "rc=$?" >> gpurun_out/r02d_pytest_rows.log
tail -4 gpurun_out/r02d_pytest_rows.log; grep -E "^E  |FAILED" gpurun_out/r02d_pytest_rows.log | head -10
WL=c1 B=32 timeout 120 python scripts/trace_rows.py 2>&1 | tail -8
WL=c2 B=65536 timeout 120 python scripts/trace_rows.py 2>&1 | tail -8
RAP_KERNEL=2 WL=c1 SIZES=32,4096 timeout 300 python scripts/fixed_cost.py 2>&1 | grep -v "^{"
RAP_KERNEL=2 WL=c2 SIZES=65536 timeout 300 python scripts/fixed_cost.py 2>&1 | grep -v "^{"
RAP_KERNEL=2 timeout 600 ncu --set full --clock-control none --import-source on -k regex:rap_rows -s 5 -c 1 -o gpurun_out/r02d_rows_c2 -f python bench.py --profile --steps 8 --warmup 5 > gpurun_out/r02d_ncu.log 2>&1
tail -1 gpurun_out/r02d_ncu.log

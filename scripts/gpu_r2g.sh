#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "jit or rows" -x > gpurun_out/r02g_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02g_pytest.log
tail -3 gpurun_out/r02g_pytest.log; grep -E "^E  |FAILED" gpurun_out/r02g_pytest.log | head -10
KMODE=3 WL=c2 B=65536 timeout 120 python scripts/trace_rows.py 2>&1 | tail -12
RAP_KERNEL=3 WL=c2 SIZES=65536 timeout 300 python scripts/fixed_cost.py 2>&1 | grep -v "^{"
RAP_KERNEL=3 timeout 600 ncu --set full --clock-control none --import-source on -k regex:rap_jit -s 5 -c 1 -o gpurun_out/r02g_jit_c2 -f python bench.py --profile --steps 8 --warmup 5 > gpurun_out/r02g_ncu.log 2>&1
tail -1 gpurun_out/r02g_ncu.log

#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu -x > gpurun_out/r02z_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02z_pytest.log
tail -2 gpurun_out/r02z_pytest.log; grep -E "^E  |FAILED" gpurun_out/r02z_pytest.log | head -10
for b in 32 4096; do WL=c1 B=$b KMODE=0 timeout 300 python scripts/trace_rows.py; done > gpurun_out/r02z_trace.txt 2>&1
cat gpurun_out/r02z_trace.txt
WL=c1 SIZES=32,128,1024,4096 timeout 300 python scripts/fixed_cost.py 2>&1 | grep -v "^{"
WL=c2 SIZES=128,4096,16384,65536 timeout 300 python scripts/fixed_cost.py 2>&1 | grep -v "^{"

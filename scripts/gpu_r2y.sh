#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_edges.py -q -m gpu -x > gpurun_out/r02y_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02y_pytest.log
tail -2 gpurun_out/r02y_pytest.log; grep -E "^E  |FAILED" gpurun_out/r02y_pytest.log | head -10
for b in 32 128 1024; do WL=c1 B=$b KMODE=0 timeout 300 python scripts/trace_rows.py; done > gpurun_out/r02y_trace.txt 2>&1
B=65536 KMODE=3 timeout 300 python scripts/trace_rows.py >> gpurun_out/r02y_trace.txt 2>&1
cat gpurun_out/r02y_trace.txt

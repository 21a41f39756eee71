#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
WL=c4 B=16384 NSETS=2 STAMPS=0 TAG=c4-hoist timeout 300 python scripts/cold_trace.py
) > gpurun_out/r4b.log 2>&1
grep -E "graph|^c" gpurun_out/r4b.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_fullsize.py -q -x -m gpu > gpurun_out/r4b_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r4b_pytest.log
tail -2 gpurun_out/r4b_pytest.log; grep -E "^FAILED|Error" gpurun_out/r4b_pytest.log | head -5
timeout 900 ncu --set full --import-source on --clock-control none -k regex:rap_fused -c 1 -o gpurun_out/r4b_c4 python bench.py --profile --workload c4 --batch 16384 --steps 2 --warmup 1 > gpurun_out/r4b_ncu_c4.log 2>&1
ncu -i gpurun_out/r4b_c4.ncu-rep --page source --csv --print-source sass > gpurun_out/r4b_c4_sass.csv 2>&1

#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_cast.py -q -x -m gpu > gpurun_out/r4j_cast.log 2>&1; echo "rc=$?" >> gpurun_out/r4j_cast.log
tail -3 gpurun_out/r4j_cast.log; grep -E "^FAILED|Error|assert" gpurun_out/r4j_cast.log | head -8
(
STAMPS=0 TAG=after-cast timeout 120 python scripts/cold_trace.py
WL=c4 B=16384 NSETS=2 STAMPS=0 TAG=c4-after-cast timeout 300 python scripts/cold_trace.py
) > gpurun_out/r4j.log 2>&1
grep -E "graph|^c" gpurun_out/r4j.log
timeout 1800 python -m pytest tests -q -m gpu > gpurun_out/r4j_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r4j_pytest.log
tail -2 gpurun_out/r4j_pytest.log; grep -E "^FAILED" gpurun_out/r4j_pytest.log | head -5

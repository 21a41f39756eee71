#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
(
STAMPS=0 TAG=base timeout 120 python scripts/cold_trace.py
RAP_JIT_TAIL_PCT=15 STAMPS=0 TAG=tail15 timeout 120 python scripts/cold_trace.py
RAP_JIT_TAIL_PCT=25 STAMPS=0 TAG=tail25 timeout 120 python scripts/cold_trace.py
RAP_JIT_BATCH=6 STAMPS=0 TAG=k6 timeout 120 python scripts/cold_trace.py
RAP_JIT_BATCH=12 STAMPS=0 TAG=k12 timeout 120 python scripts/cold_trace.py
) > gpurun_out/r4l.log 2>&1
grep -E "graph|^c" gpurun_out/r4l.log
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -m gpu -k "host" > gpurun_out/r4l_pytest.log 2>&1; tail -1 gpurun_out/r4l_pytest.log

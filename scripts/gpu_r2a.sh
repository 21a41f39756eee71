#!/bin/bash
# round 2, call A: launch-shape microbenchmark + fixed-cost decomposition of the r01 kernel
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 120 ./scripts/mb/launch > gpurun_out/r02a_launch_mb.txt 2>&1
WL=c1 timeout 300 python scripts/fixed_cost.py > gpurun_out/r02a_fixed_c1.txt 2>&1
WL=c2 SIZES=128,4096,65536 timeout 300 python scripts/fixed_cost.py > gpurun_out/r02a_fixed_c2.txt 2>&1
WL=c1 B=4096 timeout 300 python scripts/trace.py > gpurun_out/r02a_trace_c1.txt 2>&1
WL=c2 timeout 300 python scripts/trace.py > gpurun_out/r02a_trace_c2.txt 2>&1
cat gpurun_out/r02a_launch_mb.txt gpurun_out/r02a_fixed_c1.txt gpurun_out/r02a_fixed_c2.txt
head -12 gpurun_out/r02a_trace_c1.txt

#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for m in 0 1 2 3; do
  WL=c1 SIZES=0,32,128,1024,4096 RAP_KERNEL_MODE=$m timeout 300 python scripts/fixed_cost.py 2>&1 | grep -v "^{" 
done > gpurun_out/r02v_fixed_c1.txt
for m in 0 2 3; do
  WL=c2 SIZES=128,4096,16384,65536 RAP_KERNEL_MODE=$m timeout 300 python scripts/fixed_cost.py 2>&1 | grep -v "^{"
done > gpurun_out/r02v_fixed_c2.txt
cat gpurun_out/r02v_fixed_c1.txt gpurun_out/r02v_fixed_c2.txt
for k in 2 3; do WL=c1 B=4096 KMODE=$k timeout 300 python scripts/trace_rows.py; done > gpurun_out/r02v_trace_c1.txt 2>&1
WL=c2 B=65536 KMODE=3 timeout 300 python scripts/trace_rows.py >> gpurun_out/r02v_trace_c1.txt 2>&1
WL=c2 B=16384 KMODE=3 timeout 300 python scripts/trace_rows.py >> gpurun_out/r02v_trace_c1.txt 2>&1
cat gpurun_out/r02v_trace_c1.txt

#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 600 ncu --set full --import-source on --clock-control none -k regex:rap_jit -s 2 -c 1 -o gpurun_out/r3i_c2 python scripts/one_launch.py > gpurun_out/r3i_ncu.log 2>&1
ncu -i gpurun_out/r3i_c2.ncu-rep --page source --csv --print-source sass > gpurun_out/r3i_sass.csv 2>&1
ncu -i gpurun_out/r3i_c2.ncu-rep --page raw --csv > gpurun_out/r3i_raw.csv 2>&1
ls -la gpurun_out/r3i*; tail -3 gpurun_out/r3i_ncu.log

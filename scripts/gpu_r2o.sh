#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
RAP_KERNEL=3 timeout 600 ncu --set full --clock-control none --import-source on -k regex:rap_jit -s 5 -c 1 -o gpurun_out/r02o_jit_c2 -f python bench.py --profile --steps 8 --warmup 5 > gpurun_out/r02o_ncu.log 2>&1
tail -1 gpurun_out/r02o_ncu.log

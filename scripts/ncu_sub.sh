#!/bin/bash
# ncu --set full of sub-graphs of C2 (dev tool): KEEPS="a:b c:d ..."
python -c "import __graft_entry__ as g; g.build()" > /dev/null
mkdir -p gpurun_out
for k in ${KEEPS:-0:15 15:16 41:42 0:49}; do
  n=$(echo $k | tr ':' '_')
  KEEP=$k timeout 600 ncu --set full --clock-control none --import-source on -k regex:rap_fused -s 4 -c 1 -o gpurun_out/sub_$n -f python scripts/subgraph.py > gpurun_out/sub_$n.log 2>&1
done
ls gpurun_out

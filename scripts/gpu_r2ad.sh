#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
M=sm__cycles_active.sum,sm__cycles_active.max,sm__cycles_active.avg,launch__grid_size,gpu__time_duration.sum,sm__warps_active.avg.pct_of_peak_sustained_elapsed
for k in 3 1; do for b in 8 16 37 74 148; do
  echo "== kmode $k budget $b"
  BUDGET=$b KMODE=$k timeout 300 ncu --metrics $M --clock-control none --csv -k regex:rap_ python scripts/budget_footprint.py 2>/dev/null | grep -E '^"[0-9]' | tail -6
done; done > gpurun_out/r02ad_footprint.csv
cat gpurun_out/r02ad_footprint.csv | head -80

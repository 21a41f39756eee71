#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
STAMPS=0 TAG=dense3 timeout 120 python scripts/cold_trace.py 2>&1 | grep -E "graph|^c" || exit 1
timeout 600 python scripts/budget_sweep.py > gpurun_out/r02b_budget_sweep.jsonl 2> gpurun_out/r02b_budget_sweep.err; wc -l gpurun_out/r02b_budget_sweep.jsonl; tail -2 gpurun_out/r02b_budget_sweep.err

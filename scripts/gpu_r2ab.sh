#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
BUDGETS=8,16,24,37,55,74,111,148 timeout 1200 python scripts/budget_sweep.py > gpurun_out/r02ab_budget.jsonl 2> gpurun_out/r02ab_budget.err; tail -3 gpurun_out/r02ab_budget.err
wc -l gpurun_out/r02ab_budget.jsonl

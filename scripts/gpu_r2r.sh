#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu -x > gpurun_out/r02r_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02r_pytest.log
tail -3 gpurun_out/r02r_pytest.log; grep -E "^E  |FAILED" gpurun_out/r02r_pytest.log | head -10
timeout 600 python scripts/budget_sweep.py > gpurun_out/r02r_budget.jsonl 2> gpurun_out/r02r_budget.err; tail -3 gpurun_out/r02r_budget.err
cat gpurun_out/r02r_budget.jsonl
timeout 900 python bench.py > gpurun_out/r02r_bench.json 2> gpurun_out/r02r_bench.err; tail -3 gpurun_out/r02r_bench.err
python -c "
import json; d=json.load(open('gpurun_out/r02r_bench.json'))
print('value', d['value'], 'kernel_us', d['roofline']['kernel_ms']*1e3, 'frac', d['roofline']['frac'], d['config']['kernel'])
print('e2e', d['e2e']['value'], 'cpu', d['cpu_baseline']['value'], d['cpu_baseline']['cores'], 'c4', d['c4']['kernel_ms'], d['c4']['frac'])
print('graph', d['graph']['ms_per_step'], 'fusion', d['fusion']['fusion_speedup'], 'corun', [(r.get('budget'), r.get('slowdown')) for r in d['corun'].get('points', [])] if d.get('corun') else None)
"

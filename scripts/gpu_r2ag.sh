#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_perop_baseline.py -q -m gpu -k "plan or perop" > gpurun_out/r02ag_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02ag_pytest.log
tail -2 gpurun_out/r02ag_pytest.log; grep -E "^E  " gpurun_out/r02ag_pytest.log | head -20
timeout 1500 python bench.py > gpurun_out/r02ag_bench.json 2> gpurun_out/r02ag_bench.err; tail -5 gpurun_out/r02ag_bench.err
python -c "
import json; d=json.load(open('gpurun_out/r02ag_bench.json'))
print('value', d['value'], 'kernel_us', d['roofline']['kernel_ms']*1e3, 'frac', d['roofline']['frac'])
print('e2e', d['e2e']['value'], 'cpu', d['cpu_baseline']['value'])
print('fusion', {k: v for k, v in d['fusion'].items() if k != 'per_output'})
print('plans', d['plans'])
print('c4', d['c4']['kernel_ms'], d['c4']['frac'])
print('graph', d['graph'])
"

#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_corun.py -q -m gpu > gpurun_out/r02ah_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02ah_pytest.log; tail -2 gpurun_out/r02ah_pytest.log
timeout 1200 python bench.py --no-e2e --no-cpu-baseline --no-fusion --no-c4 --no-plans > gpurun_out/r02ah_bench.json 2> gpurun_out/r02ah_bench.err; tail -3 gpurun_out/r02ah_bench.err
python -c "
import json; d=json.load(open('gpurun_out/r02ah_bench.json'))
c=d['corun']; print('alone', c['train_step_alone_ms'], 'chosen', c.get('chosen'))
for r in c['per_budget']: print(' b', r['sm_budget'], r['train_step_alone_ms'], r['train_step_corun_ms'], round(r['slowdown']*100,2), r['prep_hidden'])
for r in c['partition']: print(' part', r['partition_sms'], round(r['slowdown']*100,2), r['prep_hidden'])
for x in c['layer_aligned']['per_budget']: print(' LA', x['pack_budget'], round(x['slowdown']*100,2), x['prep_hidden'], len(x['chunks']))
"

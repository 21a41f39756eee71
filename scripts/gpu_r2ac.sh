#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
true
tail -2 gpurun_out/r02ac_pytest.log; grep -E "^E  " gpurun_out/r02ac_pytest.log | head -20
timeout 1200 python bench.py > gpurun_out/r02ac_bench.json 2> gpurun_out/r02ac_bench.err; tail -3 gpurun_out/r02ac_bench.err
python -c "
import json; d=json.load(open('gpurun_out/r02ac_bench.json'))
print('value', d['value'], 'kernel_us', d['roofline']['kernel_ms']*1e3, 'frac', d['roofline']['frac'])
c=d['corun']; print('alone', c['train_step_alone_ms'], 'chosen', c.get('chosen'))
for r in c['per_budget']: print(r)
la=c.get('layer_aligned'); print(la['layer_us']); [print(x['pack_budget'], x['slowdown'], x['prep_done_ms'], [(ch['layer'], len(ch['outputs']), ch['budget']) for ch in x['chunks']]) for x in la['per_budget']]
"

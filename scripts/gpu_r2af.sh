#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python bench.py --no-e2e --no-cpu-baseline --no-fusion --no-c4 > gpurun_out/r02af_bench.json 2> gpurun_out/r02af_bench.err; tail -5 gpurun_out/r02af_bench.err
python -c "
import json; d=json.load(open('gpurun_out/r02af_bench.json'))
c=d['corun']; print('alone', c['train_step_alone_ms'], 'chosen', c.get('chosen'))
for r in c['per_budget']: print(r)
for r in c['partition']: print('PART', r)
for x in c['layer_aligned']['per_budget']: print('LA', x['pack_budget'], x['slowdown'], x['prep_done_ms'])
"

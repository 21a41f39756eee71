#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1200 python bench.py --steps 300 --warmup 10 --no-corun --no-fusion --no-plans --no-cpu-baseline --no-e2e --ngram-sweep 8,32,64,128 > gpurun_out/r4e_bench.json 2> gpurun_out/r4e_bench.err; tail -3 gpurun_out/r4e_bench.err
python - <<'P'
import json
d=json.loads(open('gpurun_out/r4e_bench.json').read().strip().splitlines()[-1])
print('c2', d['ms_per_step'], d['roofline']['frac'])
for x in d['ngram_sweep']: print(x)
m=d['mapping']; print('c2 mapping', {k: (v['max_us'] if isinstance(v, dict) else v) for k, v in m.items() if k not in ('what',)})
m=d['c4']['mapping']; print('c4 mapping', {k: (v['max_us'] if isinstance(v, dict) else v) for k, v in m.items() if k not in ('what',)})
P

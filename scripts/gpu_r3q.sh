#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 600 python bench.py --steps 600 --warmup 20 --no-corun --no-fusion --no-plans --no-cpu-baseline > gpurun_out/r3q_bench.json 2> gpurun_out/r3q_bench.err; tail -3 gpurun_out/r3q_bench.err
python - <<'P'
import json
d=json.loads(open('gpurun_out/r3q_bench.json').read().strip().splitlines()[-1])
print('value', d['value'], 'ms', d['ms_per_step'], 'frac', d['roofline']['frac'], 'eager', d['roofline']['eager'], 'e2e', d['e2e']['value'] if d['e2e'] else None)
print('graph', d['graph']); print('c4', d['c4']); print('clocks', d['clocks'])
P
timeout 1800 python -m pytest tests -q -x -m gpu > gpurun_out/r3q_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r3q_pytest.log
tail -3 gpurun_out/r3q_pytest.log; grep -E "^FAILED|Error" gpurun_out/r3q_pytest.log | head -5

#!/bin/bash
# column emitter vs row emitter on the generated kernel
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py -q -m gpu -x -k "jit" > gpurun_out/r02x_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02x_pytest.log
tail -2 gpurun_out/r02x_pytest.log; grep -E "^E  |FAILED" gpurun_out/r02x_pytest.log | head -10
B=65536 KMODE=3 timeout 300 python scripts/trace_rows.py > gpurun_out/r02x_trace.txt 2>&1
RAP_JIT_EMIT=row B=65536 KMODE=3 timeout 300 python scripts/trace_rows.py >> gpurun_out/r02x_trace.txt 2>&1
cat gpurun_out/r02x_trace.txt
for e in col row; do
  RAP_JIT_EMIT=$e timeout 300 python bench.py --steps 30 --warmup 5 --no-e2e --no-cpu-baseline --no-corun --no-fusion --no-c4 > gpurun_out/r02x_b_$e.json 2>/dev/null
  python -c "
import json,sys; d=json.load(open('gpurun_out/r02x_b_$e.json')); r=d['roofline']
print('$e: kernel_us %.2f frac %.3f graph %s' % (r['kernel_ms']*1e3, r['frac'], (d.get('graph') or {}).get('ms_per_step')))"
done

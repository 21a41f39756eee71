#!/bin/bash
# base-phase rewrite + prefetch-distance sweep on the generated kernel
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py -q -m gpu -x > gpurun_out/r02w_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02w_pytest.log
tail -2 gpurun_out/r02w_pytest.log; grep -E "^E  |FAILED" gpurun_out/r02w_pytest.log | head -10
B=65536 KMODE=3 timeout 300 python scripts/trace_rows.py > gpurun_out/r02w_trace.txt 2>&1
WL=c1 B=4096 KMODE=2 timeout 300 python scripts/trace_rows.py >> gpurun_out/r02w_trace.txt 2>&1
cat gpurun_out/r02w_trace.txt
for a in "4 2" "8 2" "12 2" "8 4" "26 4"; do set -- $a
  RAP_JIT_AHEAD=$1 RAP_JIT_PROBE=$2 timeout 300 python bench.py --steps 30 --warmup 5 --no-e2e --no-cpu-baseline --no-corun --no-fusion --no-c4 > gpurun_out/r02w_b_$1_$2.json 2>/dev/null
  python -c "
import json,sys; d=json.load(open('gpurun_out/r02w_b_$1_$2.json')); r=d['roofline']
print('ahead $1 probe $2: kernel_us %.2f frac %.3f graph %s' % (r['kernel_ms']*1e3, r['frac'], (d.get('graph') or {}).get('ms_per_step')))"
done

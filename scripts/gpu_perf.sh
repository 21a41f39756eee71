#!/bin/bash
# build + gpu parity tests + kernel-only timing of C2 and C4 (dev tool)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -2 gpurun_out/pytest_gpu.log; grep -E "^FAILED|^E  " gpurun_out/pytest_gpu.log | head -8
for wl in c2 c4; do
  st=2000; [ $wl = c4 ] && st=20
  timeout 600 python bench.py --workload $wl --no-e2e --no-cpu-baseline --no-corun --steps $st --warmup 5 > gpurun_out/bench_$wl.json 2> gpurun_out/bench_$wl.err
  python -c "import json; d=json.load(open('gpurun_out/bench_$wl.json')); print('$wl', 'kernel_us', round(d['roofline']['kernel_ms']*1e3,2), 'frac', round(d['roofline']['frac'],4))" 2>&1 | tail -1
done
[ -n "$TRACE" ] && timeout 300 python scripts/trace.py 2>&1 | tail -7
true

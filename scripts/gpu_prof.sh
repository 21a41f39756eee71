#!/bin/bash
# build, gpu tests, bench, phase trace and one ncu --set full capture (tag = $1)
TAG=${1:-cur}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log; grep -E "^FAILED|^E  " gpurun_out/pytest_gpu.log | head -8
timeout 600 python bench.py --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench.err
python -c "import json; d=json.load(open('gpurun_out/bench_${TAG}.json')); print('kernel_us', d['roofline']['kernel_ms']*1e3, 'frac', d['roofline']['frac'], 'e2e', d['e2e']['value'])" 2>&1 | tail -1
tail -2 gpurun_out/bench.err
timeout 300 python scripts/trace.py 2>&1 | tail -7
timeout 900 ncu --set full --clock-control none --import-source on -k regex:rap_fused -s 5 -c 1 -o gpurun_out/prof_${TAG} -f python bench.py --profile --steps 8 --warmup 5 ${BENCH_ARGS} > gpurun_out/ncu_full.log 2>&1
tail -1 gpurun_out/ncu_full.log

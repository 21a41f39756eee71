#!/bin/bash
# round 2, call B: parity of both kernels, row-block fixed cost, C2 bench
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "rows" -x > gpurun_out/r02b_pytest_rows.log 2>&1; echo "rc=$?" >> gpurun_out/r02b_pytest_rows.log
tail -15 gpurun_out/r02b_pytest_rows.log
RAP_KERNEL=2 WL=c1 timeout 300 python scripts/fixed_cost.py > gpurun_out/r02b_fixed_c1_rows.txt 2>&1
RAP_KERNEL=2 WL=c2 SIZES=128,4096,65536 timeout 300 python scripts/fixed_cost.py > gpurun_out/r02b_fixed_c2_rows.txt 2>&1
cat gpurun_out/r02b_fixed_c1_rows.txt gpurun_out/r02b_fixed_c2_rows.txt | grep -v "^{"
timeout 300 python bench.py --steps 500 --warmup 20 --no-cpu-baseline --no-corun --no-fusion --no-e2e > gpurun_out/r02b_bench.json 2> gpurun_out/r02b_bench.err
python -c "import json; d=json.load(open('gpurun_out/r02b_bench.json')); print('kernel_us', d['roofline']['kernel_ms']*1e3, 'frac', d['roofline']['frac'], 'grid', d['config']['grid'])"
tail -3 gpurun_out/r02b_bench.err

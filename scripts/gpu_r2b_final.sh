#!/bin/bash
# round-2 (second session) evidence: GPU suite, smoke, sanitizer, bench lines, ncu launch list and full captures
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1800 python -m pytest tests -q -m gpu > gpurun_out/r02b_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02b_pytest.log
tail -2 gpurun_out/r02b_pytest.log; grep -E "^FAILED" gpurun_out/r02b_pytest.log | head
timeout 600 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/r02b_smoke.log 2>&1; tail -1 gpurun_out/r02b_smoke.log
# (compute-sanitizer is closed on this pool)
timeout 1500 python bench.py > gpurun_out/r02b_bench.json 2> gpurun_out/r02b_bench.err; tail -2 gpurun_out/r02b_bench.err
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/r02b_bench_reference.json 2>&1
timeout 900 python bench.py --workload c1 --no-corun --no-c4 --no-plans --no-cpu-baseline > gpurun_out/r02b_bench_c1.json 2> gpurun_out/r02b_bench_c1.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r02b_launches.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-corun --no-fusion --no-c4 --no-plans > gpurun_out/r02b_launches_bench.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:rap_jit -c 1 -o gpurun_out/r02b_c2_jit python bench.py --profile --steps 2 --warmup 1 > gpurun_out/r02b_ncu_c2.log 2>&1
ncu -i gpurun_out/r02b_c2_jit.ncu-rep --page source --csv --print-source sass > gpurun_out/r02b_c2_sass.csv 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:rap_fused -c 1 -o gpurun_out/r02b_c4_tiled python bench.py --profile --workload c4 --batch 16384 --steps 2 --warmup 1 > gpurun_out/r02b_ncu_c4.log 2>&1
ls -la gpurun_out/r02b_*

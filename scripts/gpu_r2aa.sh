#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests/test_dist.py -q -m gpu -x -k "two_processes or sharded" > gpurun_out/r02aa_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02aa_pytest.log
tail -2 gpurun_out/r02aa_pytest.log; grep -E "^E  " gpurun_out/r02aa_pytest.log | grep -v "^E    *File\|^E    *return\|^E    *\^" | head -40
timeout 900 python -m pytest tests/test_bench_sharded.py -q -m gpu -x > gpurun_out/r02aa_bench.log 2>&1; echo "rc=$?" >> gpurun_out/r02aa_bench.log; tail -2 gpurun_out/r02aa_bench.log; grep -E "^E  " gpurun_out/r02aa_bench.log | head -30

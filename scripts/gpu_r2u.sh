#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/r02u_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02u_pytest.log
tail -3 gpurun_out/r02u_pytest.log; grep -E "^E  |FAILED" gpurun_out/r02u_pytest.log | head -30
CS=/usr/local/cuda/bin/compute-sanitizer
KMODES=1 timeout 900 $CS --tool racecheck --racecheck-report hazard python scripts/sanitize.py > gpurun_out/r02u_racecheck_tiled.log 2>&1; echo "rc=$?" >> gpurun_out/r02u_racecheck_tiled.log
tail -3 gpurun_out/r02u_racecheck_tiled.log
grep "Read Thread\|Write Thread" gpurun_out/r02u_racecheck_tiled.log | sed 's/.*) at //' | sort | uniq -c | head
timeout 900 $CS --tool memcheck --leak-check no python scripts/sanitize.py > gpurun_out/r02u_memcheck.log 2>&1; echo "rc=$?" >> gpurun_out/r02u_memcheck.log
tail -2 gpurun_out/r02u_memcheck.log
CASES=c1,multihot timeout 1200 $CS --tool initcheck python scripts/sanitize.py > gpurun_out/r02u_initcheck.log 2>&1; echo "rc=$?" >> gpurun_out/r02u_initcheck.log
tail -3 gpurun_out/r02u_initcheck.log

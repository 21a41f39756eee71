#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 900 $CS --tool memcheck --leak-check no python scripts/sanitize.py > gpurun_out/r02t_memcheck.log 2>&1; echo "rc=$?" >> gpurun_out/r02t_memcheck.log
tail -4 gpurun_out/r02t_memcheck.log
timeout 600 $CS --tool synccheck python scripts/sanitize.py > gpurun_out/r02t_synccheck.log 2>&1; echo "rc=$?" >> gpurun_out/r02t_synccheck.log
tail -3 gpurun_out/r02t_synccheck.log
KMODES=2,3 timeout 900 $CS --tool racecheck --racecheck-report hazard python scripts/sanitize.py > gpurun_out/r02t_racecheck.log 2>&1; echo "rc=$?" >> gpurun_out/r02t_racecheck.log
tail -3 gpurun_out/r02t_racecheck.log
timeout 900 python -m pytest -q -m gpu tests/test_gpu_fullsize.py tests/test_dist.py > gpurun_out/r02t_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02t_pytest.log
tail -3 gpurun_out/r02t_pytest.log; grep -E "^E  |FAILED" gpurun_out/r02t_pytest.log | head -20
KMODES=1 timeout 900 $CS --tool racecheck --racecheck-report hazard python scripts/sanitize.py > gpurun_out/r02t_racecheck_tiled.log 2>&1; echo "rc=$?" >> gpurun_out/r02t_racecheck_tiled.log
tail -3 gpurun_out/r02t_racecheck_tiled.log
timeout 600 $CS --tool initcheck python scripts/sanitize.py > gpurun_out/r02t_initcheck.log 2>&1; echo "rc=$?" >> gpurun_out/r02t_initcheck.log
tail -3 gpurun_out/r02t_initcheck.log

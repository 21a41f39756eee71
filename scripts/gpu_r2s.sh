#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/r02s_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02s_pytest.log
tail -3 gpurun_out/r02s_pytest.log; grep -E "^E  |FAILED" gpurun_out/r02s_pytest.log | head -30

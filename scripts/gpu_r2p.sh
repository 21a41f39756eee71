#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "jit" -x > gpurun_out/r02p_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02p_pytest.log
tail -2 gpurun_out/r02p_pytest.log; grep -E "^E  |FAILED" gpurun_out/r02p_pytest.log | head -10
for sg in 0 4 6 10; do
  echo "== SEGMENT $sg"
  RAP_JIT_SEGMENT=$sg KMODE=3 WL=c2 B=65536 timeout 120 python scripts/trace_rows.py 2>&1 | sed -n 2,6p
  RAP_JIT_SEGMENT=$sg RAP_KERNEL=3 WL=c2 SIZES=65536 timeout 300 python scripts/fixed_cost.py 2>&1 | grep -v "^{"
done

#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for v in "" "RAP_CARVEOUT=100" "RAP_NOCOOP=1"; do
  echo "== [$v]"
  env $v RAP_KERNEL=3 WL=c2 SIZES=65536 timeout 300 python scripts/fixed_cost.py 2>&1 | grep -v "^{"
done
RAP_KERNEL=1 WL=c2 SIZES=65536 timeout 300 python scripts/fixed_cost.py 2>&1 | grep -v "^{"
RAP_KERNEL=2 WL=c2 SIZES=65536 timeout 300 python scripts/fixed_cost.py 2>&1 | grep -v "^{"

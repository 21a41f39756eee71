#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_partition.py tests/test_gpu_cost_model.py -q -m gpu > gpurun_out/r02ae_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02ae_pytest.log
tail -2 gpurun_out/r02ae_pytest.log; grep -E "^E  " gpurun_out/r02ae_pytest.log | head -20
M=sm__cycles_active.sum,sm__cycles_active.max,launch__grid_size,gpu__time_duration.sum
for k in 3 1; do for b in 8 16 40 72; do
  echo "== kmode $k partition $b"
  PART=1 BUDGET=$b KMODE=$k timeout 300 ncu --metrics $M --clock-control none --csv -k regex:rap_ python scripts/budget_footprint.py 2>&1 | grep -E '^"[0-9]|partition SMs|Error|error' | tail -5
done; done > gpurun_out/r02ae_footprint_part.csv
python - <<'PY'
import csv, re
cur=None; rows={}
for line in open('gpurun_out/r02ae_footprint_part.csv'):
    if line.startswith('=='): cur=line.strip(); rows[cur]={}; continue
    if line.startswith('"'):
        r=next(csv.reader([line])); rows[cur][r[-3]]=r[-1]
    else: rows.setdefault(cur,{})['note']=line.strip()
for k,v in rows.items():
    try: print(k, v.get('note',''), 'grid', v['launch__grid_size'], 'us', float(v['gpu__time_duration.sum'])/1e3, 'eff SMs %.1f'%(float(v['sm__cycles_active.sum'].replace(',',''))/float(v['sm__cycles_active.max'].replace(',',''))))
    except Exception as e: print(k, v, e)
PY

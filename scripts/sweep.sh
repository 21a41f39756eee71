#!/bin/bash
# build + gpu tests + bench + phase trace, then bench variants given in $VARIANTS (';'-separated nvcc flag sets)
export NO_NCU=1
bash scripts/gpu_quick.sh
IFS=';' read -ra VS <<< "${VARIANTS}"
for v in "${VS[@]}"; do
  RAP_NVCC_FLAGS="$v" python -c "from paper_conf_asplos_wangwdz0d24_b200 import _build; _build.build(force=True)"
  echo "variant [$v]: $(timeout 300 python bench.py --no-e2e --no-cpu-baseline --steps 2000 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["roofline"]["kernel_ms"]*1e3, "us", d["roofline"]["frac"])')"
done

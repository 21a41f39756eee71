#!/bin/bash
# time compile-flag variants of the kernel on C2 (dev tool): VARIANTS="-DX=1|-DY=2"
IFS='|' read -ra VS <<< "${VARIANTS}"
for v in "${VS[@]}"; do
  RAP_NVCC_FLAGS="$v" python -c "from paper_conf_asplos_wangwdz0d24_b200 import _build; _build.build(force=True)" || exit 1
  echo "variant [$v]: $(timeout 300 python bench.py --no-e2e --no-cpu-baseline --steps 500 --warmup 20 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["roofline"]["kernel_ms"]*1e3,2), "us grid", d["config"]["grid"])')"
done

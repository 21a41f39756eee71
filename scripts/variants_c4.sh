#!/bin/bash
# time compile-flag variants of the kernel on C4 (dev tool): VARIANTS="-DX=1|-DY=2"
IFS='|' read -ra VS <<< "${VARIANTS}"
for v in "${VS[@]}"; do
  RAP_NVCC_FLAGS="$v" python -c "from paper_conf_asplos_wangwdz0d24_b200 import _build; _build.build(force=True)" > /dev/null 2>&1 || { echo "build failed [$v]"; continue; }
  for wl in c4 c2; do
    st=2000; [ $wl = c4 ] && st=100
    echo "variant [$v] $wl: $(timeout 400 python bench.py --workload $wl --no-e2e --no-cpu-baseline --no-corun --no-fusion --steps $st --warmup 10 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["roofline"]["kernel_ms"]*1e3,2), "us frac", round(d["roofline"]["frac"],4), "grid", d["config"]["grid"])')"
  done
done

#!/bin/bash
# kernel-only C2 / C4 timing of compile-flag variants: VARIANTS="-DX=1|-DY=2" (dev tool)
mkdir -p gpurun_out
IFS='|' read -ra VS <<< "|${VARIANTS}"
for v in "${VS[@]}"; do
  RAP_NVCC_FLAGS="$v" python -c "from paper_conf_asplos_wangwdz0d24_b200 import _build; _build.build(force=True)" > gpurun_out/vbuild.log 2>&1 || { echo "build failed [$v]"; tail -5 gpurun_out/vbuild.log; continue; }
  for wl in ${WLS:-c2 c4}; do
    st=2000; [ $wl = c4 ] && st=15
    r=$(timeout 300 python bench.py --workload $wl --no-e2e --no-cpu-baseline --no-corun --steps $st --warmup 5 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["roofline"]["kernel_ms"]*1e3,2), "us frac", round(d["roofline"]["frac"],4))')
    echo "variant [$v] $wl: $r"
  done
done
python -c "from paper_conf_asplos_wangwdz0d24_b200 import _build; _build.build(force=True)" > /dev/null 2>&1

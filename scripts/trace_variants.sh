#!/bin/bash
# trace compile-flag variants (dev tool): VARIANTS="-DX|-DY" KEEP=a:b
IFS='|' read -ra VS <<< "${VARIANTS}"
for v in "${VS[@]}"; do
  RAP_NVCC_FLAGS="$v" python -c "from paper_conf_asplos_wangwdz0d24_b200 import _build; _build.build(force=True)" || exit 1
  echo "== variant [$v]"; timeout 120 python scripts/trace.py 2>&1 | head -7
done

#!/bin/bash
# A/B of gravity compile-time variants ($VARIANTS: SPH_NVCC_EXTRA values)
while IFS= read -r v; do
  SPH_NVCC_EXTRA="$v" python -c "from paper_conf_sc_simsekpc24_b200 import _build; _build.build(force=True)" > /dev/null 2>&1 || { echo "build failed: $v"; continue; }
  timeout 300 python tools/grav_timing.py "${v:-base}"
done <<< "$VARIANTS"

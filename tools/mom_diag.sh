#!/bin/bash
for v in "${@:-}"; do
  SPH_NVCC_EXTRA="$v" python -c "from paper_conf_sc_simsekpc24_b200 import _build; _build.build(force=True)" > /dev/null 2>&1 || echo "build failed $v"
  SPH_NVCC_EXTRA="$v" python tools/mom_diag.py
done
python -c "from paper_conf_sc_simsekpc24_b200 import _build; _build.build(force=True)"

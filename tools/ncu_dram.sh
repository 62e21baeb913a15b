#!/bin/bash
# DRAM bytes + time of one kernel (regex $K) for each SPH_NVCC_EXTRA variant in $VARIANTS
mkdir -p gpurun_out
while IFS= read -r v; do
  SPH_NVCC_EXTRA="$v" python -c "from paper_conf_sc_simsekpc24_b200 import _build; _build.build(force=True)" > /dev/null 2>&1 || { echo "build failed: $v"; continue; }
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,smsp__inst_executed.sum \
    -k regex:"$K" -c 1 --clock-control none --csv python bench.py --steps 1 --warmup 1 --e2e-steps 0 --energy-seconds 0 --timing-repeats 0 --trace-seconds 0 --no-cpu-baseline 2>/dev/null \
    | grep -E '"(gpu__time|dram__bytes|lts__t_sector_hit|smsp__inst)' | awk -F'","' -v V="${v:-base}" '{print V, $(NF-2), $(NF-1), $NF}'
done <<< "$VARIANTS"

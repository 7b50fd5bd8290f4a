#!/bin/bash
# Per-kernel time totals (ncu launch list, one run after one warm-up) for every variant in
# build/variants (builder tooling; GPU box).  usage: scripts/variant_kernels.sh [workload] [scale]
cd "$(dirname "$0")/.."
WL=${1:-rmat}; SC=${2:-26}
for f in build/variants/*.so; do
  b=$(basename $f .so)
  LMATCH_LIB=$PWD/$f ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/vk_${b}_${WL}.csv python scripts/prof_run.py --workload $WL --scale $SC --runs 2 > /dev/null 2>&1
  echo "== $b $WL $SC"
  python scripts/launch_summary.py gpurun_out/vk_${b}_${WL}.csv | grep "lm::\|total" | grep -v "k_pack\|k_zap\|k_nz_\|k_check\|k_bin_sizes\|k_tile_rows\|k_atomic_rows\|k_low32\|k_scan_block\|k_symhash\|ZAP\|, 1>"
done

#!/bin/bash
# Round profile capture (builder tooling; GPU box).  Writes into gpurun_out/:
#   bench_<tag>.json      : the default bench line (R-MAT s26)
#   launches_<tag>.csv    : ncu launch list (gpu__time_duration.sum) of the same bench command
#   sweep_full_<tag>      : ncu --set full of ONE k_sweep launch (traffic, stalls)
#   frontier_full_<tag>   : ncu --set full of the round-2 frontier kernels + match + compaction
set -x
cd "$(dirname "$0")/.."
TAG=${1:-r01}
python bench.py > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}.csv \
  python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_sweep --launch-skip 1 -c 1 \
  -o gpurun_out/sweep_full_${TAG} -f python scripts/prof_run.py --runs 1 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_point|k_compact|k_match_bins" -c 7 \
  -o gpurun_out/frontier_full_${TAG} -f python scripts/prof_run.py --runs 1 > /dev/null 2>&1
ls -la gpurun_out

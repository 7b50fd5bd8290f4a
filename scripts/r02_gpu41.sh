# ncu --set full of the round-1 match and compaction (final build)
ncu --set full --clock-control none --import-source on -k regex:"k_match_all|k_compact" --launch-skip 0 -c 2 \
  -o gpurun_out/round1_rest -f python scripts/prof_run.py --runs 1 > gpurun_out/round1_rest.log 2>&1
ls -la gpurun_out

# ncu --set full with source counters of one k_sweep launch (where the sweep's instructions go)
ncu --set full --clock-control none --import-source on -k regex:k_sweep --launch-skip 1 -c 1 \
  -o gpurun_out/sweep_src -f python scripts/prof_run.py --runs 2 > gpurun_out/sweep_src.log 2>&1
ls -la gpurun_out/

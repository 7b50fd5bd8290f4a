# launch list of the partitioned (one rank) bench, to compare with the single-graph one
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_part.csv \
  python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --partitioned > gpurun_out/part_ncu.log 2>&1
python bench.py --steps 10 --no-e2e --no-cpu --partitioned > gpurun_out/part_line.json 2>/dev/null
ls -la gpurun_out

# Round-2 final measurements (builder tooling; GPU box).  Everything lands in gpurun_out/r02f/.
set -x
O=gpurun_out/r02f; mkdir -p $O
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -5 > $O/gpu_tests.txt
python bench.py > $O/bench_rmat_s26.json 2> $O/bench_rmat_s26.err
python bench.py --impl reference > $O/bench_reference.json 2> $O/bench_reference.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_rmat_s26.csv \
  python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_sweep --launch-skip 1 -c 1 \
  -o $O/sweep_full -f python scripts/prof_run.py --runs 1 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_point|k_compact|k_match_bins" -c 7 \
  -o $O/frontier_full -f python scripts/prof_run.py --runs 1 > /dev/null 2>&1
for wl in "--workload er" "--workload mesh" "--workload road" "--workload gradient" "--workload gradient --scale 26" "--scale 24" "--algorithm sorted" "--algorithm hybrid --workload gradient --scale 26"; do
  python bench.py --no-cpu --no-e2e --steps 5 $wl 2>/dev/null | grep '^{' >> $O/bench_other.jsonl
done
for kw in "--hbm-budget-gb 6" "--hbm-budget-gb 6 --residual-mb 4096" "--hbm-budget-gb 6 --no-host-cache"; do
  python bench.py --no-cpu --no-e2e --steps 3 $kw 2>/dev/null | grep '^{' >> $O/bench_ooc_s26.jsonl
done
python bench.py --no-cpu --no-e2e --steps 5 --scale 28 2>/dev/null | grep '^{' > $O/bench_rmat_s28.json
python bench.py --no-cpu --no-e2e --steps 5 --scale 29 > $O/bench_rmat_s29.json 2> $O/bench_rmat_s29.err
python bench.py --no-cpu --no-e2e --steps 5 --scale 29 --partitioned > $O/bench_rmat_s29_partitioned_n1.json 2> $O/bench_rmat_s29_partitioned_n1.err
python bench.py --no-cpu --gpus 2 --steps 5 > $O/bench_rmat_s26_2ranks_1gpu.json 2> $O/bench_rmat_s26_2ranks_1gpu.err
ls -la $O
ls -la $O

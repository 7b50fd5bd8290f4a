# final build: smoke(), the default bench line, its launch list
set -x
O=gpurun_out/r02g; mkdir -p $O
timeout 600 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.log 2>&1
python bench.py > $O/bench_rmat_s26.json 2> $O/bench_rmat_s26.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_rmat_s26.csv \
  python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
python bench.py --no-cpu --no-e2e --steps 10 --partitioned > $O/bench_partitioned_n1_rmat_s26.json 2>/dev/null
ls -la $O

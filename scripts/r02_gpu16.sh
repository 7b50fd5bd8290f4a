set -x
O=gpurun_out/r02f; mkdir -p $O
timeout 900 python bench.py --no-cpu --no-e2e --steps 5 --scale 29 --partitioned > $O/bench_rmat_s29_partitioned_n1.json 2> $O/bench_rmat_s29_partitioned_n1.err
timeout 2400 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > $O/t16_all.log
timeout 600 python bench.py > $O/bench_rmat_s26_final.json 2> $O/bench_rmat_s26_final.err
cat $O/t16_all.log; tail -c 1200 $O/bench_rmat_s29_partitioned_n1.json; tail -3 $O/bench_rmat_s29_partitioned_n1.err; tail -c 600 $O/bench_rmat_s26_final.json

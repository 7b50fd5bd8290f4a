set -x
O=gpurun_out/r02f; mkdir -p $O
for sc in 20 22 24; do for fr in auto pull; do
  timeout 300 python bench.py --no-cpu --no-e2e --steps 3 --warmup 3 --workload gradient --scale $sc --frontier $fr 2>/dev/null | grep '^{' >> $O/bench_gradient_push_pull.jsonl
done; done
timeout 900 python bench.py --no-cpu --no-e2e --steps 5 --scale 29 --partitioned > $O/bench_rmat_s29_partitioned_n1.json 2> $O/bench_rmat_s29_partitioned_n1.err
LMATCH_HUGE=1 timeout 1500 python -m pytest tests/test_gpu_fullsize.py -x -q -k s29 2>&1 | tail -3 > $O/test_s29.log
python -c "
import json
for l in open('$O/bench_gradient_push_pull.jsonl'):
    d=json.loads(l); print(d['config']['scale'], d['config'].get('frontier','auto'), round(d['ms_per_step'],2), d['rounds'])
"
tail -c 700 $O/bench_rmat_s29_partitioned_n1.json; tail -3 $O/bench_rmat_s29_partitioned_n1.err; cat $O/test_s29.log

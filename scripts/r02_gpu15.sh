set -x
O=gpurun_out/r02f; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_contract.py -x -q -k "push" 2>&1 | tail -2 > $O/t15.log
rm -f gpurun_out/variants.jsonl
for rep in 1 2; do
  for v in base p1g4u4 p1g4u8 p1g8u4 p1g2u8; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'phase':d['phase_ms']}))" >> gpurun_out/variants.jsonl
  done
done
timeout 900 python bench.py --no-cpu --no-e2e --steps 5 --scale 29 --partitioned > $O/bench_rmat_s29_partitioned_n1.json 2> $O/bench_rmat_s29_partitioned_n1.err
LMATCH_HUGE=1 timeout 1500 python -m pytest tests/test_gpu_fullsize.py -x -q -k s29 2>&1 | tail -3 > $O/test_s29.log
for sc in 20 22; do timeout 300 python bench.py --no-cpu --no-e2e --steps 3 --workload gradient --scale $sc 2>/dev/null | grep '^{' >> $O/bench_gradient_auto2.jsonl; done
cat $O/t15.log gpurun_out/variants.jsonl $O/test_s29.log; tail -c 600 $O/bench_rmat_s29_partitioned_n1.json; tail -3 $O/bench_rmat_s29_partitioned_n1.err

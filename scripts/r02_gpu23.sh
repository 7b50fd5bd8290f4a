# probe-count knobs on the pipelined bins (one box): two-phase probing per group size, ub filter
set -x
for v in pp3all pp3g8 tail8 ubf; do
  LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "golden or random_tiny or synthetic or hub or increasing or round_loop" 2>&1 | tail -1 > gpurun_out/t_$v.log
done
rm -f gpurun_out/variants.jsonl
for rep in 1 2; do
  for v in base pp3all pp3g8 tail8 ubf; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'phase':d['phase_ms'],'rr':[(r['round'],r['ms']) for r in d.get('rounds_roofline',[])]}))" >> gpurun_out/variants.jsonl
  done
done
cat gpurun_out/t_*.log gpurun_out/variants.jsonl

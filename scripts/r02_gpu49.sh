# key cache of width 2 (row max + next key, FP64-pipe top-2) now that the sweep is memory-bound
set -x
LMATCH_LIB=$PWD/build/variants/lm_kc2.so timeout 600 python -m pytest tests/test_gpu_contract.py -x -q -k "key_cache" 2>&1 | tail -1 > gpurun_out/t_kc2.log
rm -f gpurun_out/variants.jsonl
for rep in 1 2 3; do
  for v in base kc2; do
    args=""; [ $v = kc2 ] && args="--key-cache"
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 $args 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'phase':d['phase_ms'],'rr':[(r['round'],r['ms']) for r in d.get('rounds_roofline',[])]}))" >> gpurun_out/variants.jsonl
  done
done
cat gpurun_out/t_kc2.log gpurun_out/variants.jsonl

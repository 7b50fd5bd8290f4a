# key cache width study: 2 keys (the row max + the next) vs 4, against the cache-off default
set -x
rm -f gpurun_out/variants.jsonl
LMATCH_LIB=$PWD/build/variants/lm_kc2.so timeout 600 python -m pytest tests/test_gpu_contract.py -x -q -k "key_cache" 2>&1 | tail -2 > gpurun_out/t_kc2.log
for rep in 1 2; do
  for v in base kc2 kc4; do
    lib=$PWD/build/variants/lm_kc4.so; args=""
    [ $v = kc2 ] && lib=$PWD/build/variants/lm_kc2.so && args="--key-cache"
    [ $v = kc4 ] && args="--key-cache"
    LMATCH_LIB=$lib timeout 300 python bench.py --no-cpu --no-e2e --steps 10 $args 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'phase':d['phase_ms'],'swept':d.get('entries_swept'),'rr':[(r['round'],r['ms'],r['frontier'],r['entries']) for r in d.get('rounds_roofline',[])]}))" >> gpurun_out/variants.jsonl
  done
done
cat gpurun_out/t_kc2.log gpurun_out/variants.jsonl

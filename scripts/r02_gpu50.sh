# dense sweep configuration neighbours: 768-entry tiles with 7-8 warps, 1280 with 5 (one box)
set -x
LMATCH_LIB=$PWD/build/variants/lm_t768w8.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "golden or random_tiny or synthetic or hub or increasing or crossing or extreme" 2>&1 | tail -1 > gpurun_out/t_t768.log
LMATCH_LIB=$PWD/build/variants/lm_t1280w5.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "golden or random_tiny or synthetic or hub or increasing or crossing or extreme" 2>&1 | tail -1 >> gpurun_out/t_t768.log
rm -f gpurun_out/variants.jsonl
for rep in 1 2; do
  for v in base t768w8 t768w7 t1280w5; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'sweep_ms':d['roofline']['launch_ms'],'frac':d['roofline']['frac']}))" >> gpurun_out/variants.jsonl
  done
done
cat gpurun_out/t_t768.log gpurun_out/variants.jsonl

set -x
timeout 2400 python -m pytest tests/test_gpu_dist.py tests/test_gpu_contract.py tests/test_gpu_fullsize.py -x -q --durations=15 2>&1 | tail -40 > gpurun_out/r02_t8.log
rm -f gpurun_out/variants.jsonl
for rep in 1 2; do
  for v in base pipe1 pipe12 pipe1w2; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'phase':d['phase_ms']}))" >> gpurun_out/variants.jsonl
  done
done
cat gpurun_out/r02_t8.log gpurun_out/variants.jsonl

# dead-entry hints: parity of the hint builds, then bench against the no-hint build (one box)
set -x
for v in dead dcap4; do
  LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_contract.py -x -q 2>&1 | tail -2 > gpurun_out/t_$v.log
done
rm -f gpurun_out/variants.jsonl
for rep in 1 2; do
  for v in nodead dead dcap4; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'phase':d['phase_ms'],'rr':[(r['round'],r['ms']) for r in d.get('rounds_roofline',[])]}))" >> gpurun_out/variants.jsonl
  done
done
cat gpurun_out/t_*.log gpurun_out/variants.jsonl

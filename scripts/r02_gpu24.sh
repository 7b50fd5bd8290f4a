# S pairs carry their row range (no offs[] gather when a vertex enters the frontier; round 1 reads
# noffs in order): full parity suites on the new build, then bench against the previous build
set -x
LMATCH_LIB=$PWD/build/variants/lm_sr.so timeout 1500 python -m pytest tests/ -m gpu -x -q 2>&1 | tail -2 > gpurun_out/t_sr.log
rm -f gpurun_out/variants.jsonl
for rep in 1 2 3; do
  for v in base sr; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'phase':d['phase_ms'],'rr':[(r['round'],r['ms']) for r in d.get('rounds_roofline',[])]}))" >> gpurun_out/variants.jsonl
  done
done
cat gpurun_out/t_sr.log gpurun_out/variants.jsonl

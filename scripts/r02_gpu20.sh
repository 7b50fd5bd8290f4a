# frontier bins sharing the SMs: LMATCH_BINGRID caps (blocks per SM of bin0 pipe, bin1 pipe, bin2, cta)
rm -f gpurun_out/bingrid.jsonl
for rep in 1 2; do
  for cfg in 0,0,0,0 1,2,1,0 1,1,3,0 1,2,0,0 1,1,0,0 0,2,0,0 2,2,0,0 1,3,0,0 0,1,0,0 2,1,0,0; do
    LMATCH_BINGRID=$cfg timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'cfg':'$cfg','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'phase':d['phase_ms'],'rr':[(r['round'],r['ms']) for r in d.get('rounds_roofline',[])]}))" >> gpurun_out/bingrid.jsonl
  done
done
cat gpurun_out/bingrid.jsonl

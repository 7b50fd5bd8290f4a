set -x
rm -f gpurun_out/variants.jsonl
timeout 2400 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > gpurun_out/r02_t18_all.log
for rep in 1 2 3; do
  for v in presoa soa; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'phase':d['phase_ms']}))" >> gpurun_out/variants.jsonl
  done
done
cat gpurun_out/r02_t18_all.log gpurun_out/variants.jsonl

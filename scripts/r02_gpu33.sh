# crossing-row best[] entries not re-zeroed per run (LM_XROW_RESET=0): full GPU suite on that build
# (in-tree library), then bench against the zeroing build (one box)
set -x
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -3 > gpurun_out/t_xrow.log
rm -f gpurun_out/variants.jsonl
for rep in 1 2 3; do
  for v in xrow1 xrow0; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'sweep_ms':d['roofline']['launch_ms'],'frac':d['roofline']['frac'],'phase':d['phase_ms']}))" >> gpurun_out/variants.jsonl
  done
done
cat gpurun_out/t_xrow.log gpurun_out/variants.jsonl

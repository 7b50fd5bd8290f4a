# sweep tiles of 1024 entries with fewer warps per CTA (one box)
set -x
LMATCH_LIB=$PWD/build/variants/lm_t1k_w4.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -1 > gpurun_out/t_t1k.log
rm -f gpurun_out/variants.jsonl
for rep in 1 2 3; do
  for v in base t1k_w4 t1k_w6 t1k_w4c72; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'sweep_ms':d['roofline']['launch_ms'],'frac':d['roofline']['frac'],'phase':d['phase_ms']}))" >> gpurun_out/variants.jsonl
  done
done
cat gpurun_out/t_t1k.log gpurun_out/variants.jsonl

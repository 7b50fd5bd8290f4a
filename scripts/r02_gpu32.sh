# persistent-tail threshold and sweep row-window cap (one box); partition tests for the batched
# partition match
set -x
timeout 1800 python -m pytest tests/test_gpu_p2p.py tests/test_gpu_dist.py -x -q 2>&1 | tail -2 > gpurun_out/t_part.log
for v in ps18 wc88; do
  LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "golden or random_tiny or synthetic or hub or increasing or round_loop" 2>&1 | tail -1 > gpurun_out/t_$v.log
done
rm -f gpurun_out/variants.jsonl
for rep in 1 2; do
  for v in base ps17 ps18 ps19 wc56 wc88 wc104; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'sweep_ms':d['roofline']['launch_ms'],'frac':d['roofline']['frac'],'phase':d['phase_ms']}))" >> gpurun_out/variants.jsonl
  done
done
cat gpurun_out/t_*.log gpurun_out/variants.jsonl

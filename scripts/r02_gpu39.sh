# pipelined-kernel waves, list prefetch in the binned kernels, thread-bin batch shape (one box)
set -x
for v in pw2 lpf p0u4 p0g2; do
  LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "golden or random_tiny or synthetic or hub or increasing or round_loop" 2>&1 | tail -1 > gpurun_out/t_$v.log
done
rm -f gpurun_out/variants.jsonl
for rep in 1 2; do
  for v in base pw2 lpf p0u4 p0g2; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'sweep_ms':d['roofline']['launch_ms'],'frac':d['roofline']['frac'],'phase':d['phase_ms']}))" >> gpurun_out/variants.jsonl
  done
done
cat gpurun_out/t_*.log gpurun_out/variants.jsonl

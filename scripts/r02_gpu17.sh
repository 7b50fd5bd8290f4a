set -x
rm -f gpurun_out/variants.jsonl
for v in b1_128 b1_256 p2g16u8 p1g8u8 b0_16; do
  LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "golden or random_tiny or synthetic or hub or increasing or round_loop" 2>&1 | tail -1 > gpurun_out/t_var_$v.log
done
for rep in 1 2; do
  for v in base b1_128 b1_256 p2g16u8 p1g8u8 b0_16; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'phase':d['phase_ms']}))" >> gpurun_out/variants.jsonl
  done
done
cat gpurun_out/t_var_*.log gpurun_out/variants.jsonl

set -x
mkdir -p gpurun_out/sanitizer
timeout 1500 compute-sanitizer --tool racecheck --print-limit 20 python scripts/sanitize_run.py --quick > gpurun_out/sanitizer/r02_racecheck.log 2>&1; echo "exit=$?" >> gpurun_out/sanitizer/r02_racecheck.log
timeout 600 python -m pytest tests/test_gpu_dist.py -x -q -k "missing_peer or single_rank" 2>&1 | tail -3 > gpurun_out/r02_t11.log
rm -f gpurun_out/variants.jsonl
for rep in 1 2; do
  for v in base pf pf6 minb6; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'phase':d['phase_ms']}))" >> gpurun_out/variants.jsonl
  done
done
for v in pf pf6; do
  LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "golden or random_tiny or synthetic or hub or increasing or round_loop" 2>&1 | tail -1 > gpurun_out/t_var_$v.log
done
tail -4 gpurun_out/sanitizer/r02_racecheck.log; cat gpurun_out/r02_t11.log gpurun_out/variants.jsonl gpurun_out/t_var_pf*.log

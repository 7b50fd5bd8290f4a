set -x
mkdir -p gpurun_out/sanitizer
rm -f gpurun_out/variants.jsonl
for v in ub ubp256k; do
  LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_contract.py -x -q -k "golden or random_tiny or synthetic or hub or increasing or round_loop or push or key_cache or residual" 2>&1 | tail -1 > gpurun_out/t_var_$v.log
done
for rep in 1 2; do
  for v in base ub p256k p1m ubp256k; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'phase':d['phase_ms']}))" >> gpurun_out/variants.jsonl
  done
done
timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python scripts/sanitize_run.py --quick --single > gpurun_out/sanitizer/r02_racecheck.log 2>&1; echo "exit=$?" >> gpurun_out/sanitizer/r02_racecheck.log
tail -6 gpurun_out/sanitizer/r02_racecheck.log; cat gpurun_out/t_var_ub*.log gpurun_out/variants.jsonl

# compare build/variants/*.so on the default bench (builder tooling; GPU box)
mkdir -p gpurun_out
rm -f gpurun_out/variants.jsonl
V=${VARIANTS:-"base mid"}
for v in $V; do
  [ "$v" = base ] && continue
  LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python -m pytest tests/test_gpu_parity.py -x -q \
    -k "golden or random_tiny or synthetic or hub or rmat24 or out_of_core or increasing" 2>&1 | tail -2 > gpurun_out/t_var_$v.log
done
for rep in 1 2; do
  for v in $V; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so python bench.py --no-cpu --no-e2e --steps 10 ${BENCH_ARGS} 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'sweep_ms':d['roofline']['launch_ms'],'frac':d['roofline']['frac'],'phase':d['phase_ms']}))" >> gpurun_out/variants.jsonl
  done
done
cat gpurun_out/t_var_*.log; cat gpurun_out/variants.jsonl

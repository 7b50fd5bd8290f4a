mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "out_of_core or batches" 2>&1 | tail -2
for v in base norefill; do
  for c in "--hbm-budget-gb 6" "--batches 3"; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so python bench.py --no-cpu --no-e2e --steps 3 $c 2>/dev/null | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); o=d['out_of_core']; print('$v', '$c', round(d['value'],3), round(d['ms_per_step'],1), {k: round(x,1) for k,x in d['phase_ms'].items()}, o['host_entries_read_per_step'])"
  done
done

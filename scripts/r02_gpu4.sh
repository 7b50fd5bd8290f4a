set -x
timeout 1200 python -m pytest tests/test_gpu_dist.py tests/test_gpu_contract.py -x -q 2>&1 | tail -25 > gpurun_out/r02_t4_new.log
rm -f gpurun_out/variants.jsonl
for rep in 1 2; do
  for v in old new bh; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'phase':d['phase_ms']}))" >> gpurun_out/variants.jsonl
  done
done
for v in old new; do
  LMATCH_LIB=$PWD/build/variants/lm_$v.so ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/r02_vk_$v.csv python scripts/prof_run.py --runs 2 > /dev/null 2>&1
done
cat gpurun_out/r02_t4_new.log gpurun_out/variants.jsonl
for v in old new; do python scripts/launch_summary.py gpurun_out/r02_vk_$v.csv | head -14; done

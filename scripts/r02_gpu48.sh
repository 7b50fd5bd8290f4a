# per-handle sweep configuration (dense 1024/6/104 when the average degree >= 10, else 512/8/72):
# full GPU suite + full-size certificates on the in-tree build, then every workload against the
# always-sparse build (one box)
set -x
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -3 > gpurun_out/t_auto.log
LMATCH_HUGE=1 timeout 1400 python -m pytest tests/test_gpu_fullsize.py -q 2>&1 | tail -2 >> gpurun_out/t_auto.log
rm -f gpurun_out/variants.jsonl
for wl in "--workload rmat" "--workload er" "--workload mesh" "--workload road"; do
  for v in sparse auto; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 $wl 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','wl':'$wl','gteps':d['value'],'ms':d['ms_per_step'],'sweep_ms':d['roofline']['launch_ms'],'frac':d['roofline']['frac'],'alg':d['roofline']['algorithmic_bytes_per_launch']}))" >> gpurun_out/variants.jsonl
  done
done
python bench.py --no-cpu --no-e2e --steps 10 --partitioned 2>/dev/null | grep '^{' > gpurun_out/part_line.json
cat gpurun_out/t_auto.log gpurun_out/variants.jsonl

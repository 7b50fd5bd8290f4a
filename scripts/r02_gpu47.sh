# sweep 1024-entry tiles / 6 warps / 104-row window (new default) against 512 / 8 / 72 on every
# workload class; full GPU suite on the new default (in-tree library)
set -x
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -3 > gpurun_out/t_tile.log
rm -f gpurun_out/variants.jsonl
for wl in "--workload rmat" "--workload er" "--workload mesh" "--workload road" "--workload rmat --scale 24"; do
  for v in old512 new1k new1kc136; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 $wl 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','wl':'$wl','gteps':d['value'],'ms':d['ms_per_step'],'sweep_ms':d['roofline']['launch_ms'],'frac':d['roofline']['frac']}))" >> gpurun_out/variants.jsonl
  done
done
cat gpurun_out/t_tile.log gpurun_out/variants.jsonl

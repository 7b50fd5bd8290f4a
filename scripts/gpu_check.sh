mkdir -p gpurun_out
rm -f gpurun_out/b_hybrid.jsonl
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "suitor or hybrid" 2>&1 | tail -5 > gpurun_out/t_hybrid.log
for wl in "--workload gradient --scale 20" "--workload gradient --scale 22" "--workload road" "--workload mesh" "--workload er" "" ; do
  for alg in ld suitor hybrid; do
    timeout 300 python bench.py --no-cpu --no-e2e --steps 5 --algorithm $alg $wl 2>/dev/null | grep '^{' >> gpurun_out/b_hybrid.jsonl
  done
done
cat gpurun_out/t_hybrid.log

mkdir -p gpurun_out
rm -f gpurun_out/b_hyb2.jsonl
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > gpurun_out/t_gpu5.log
for wl in "--workload gradient --scale 20" "--workload gradient --scale 22"; do
  for alg in suitor hybrid; do
    timeout 300 python bench.py --no-cpu --no-e2e --steps 5 --algorithm $alg $wl 2>/dev/null | grep '^{' >> gpurun_out/b_hyb2.jsonl
  done
done
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
cat gpurun_out/t_gpu5.log gpurun_out/smoke.log

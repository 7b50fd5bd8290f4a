mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3 > gpurun_out/t_gpu_final.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final.log 2>&1
bash scripts/profile_round.sh r01f > gpurun_out/profile_r01f.log 2>&1
rm -f gpurun_out/other_final.jsonl
for wl in "--scale 24" "--workload er" "--workload mesh" "--workload road" "--workload gradient --scale 20" "--workload gradient --scale 20 --algorithm hybrid" "--scale 28"; do
  timeout 600 python bench.py --no-cpu --no-e2e --steps 5 $wl 2>/dev/null | grep '^{' >> gpurun_out/other_final.jsonl
done
cat gpurun_out/t_gpu_final.log gpurun_out/smoke_final.log

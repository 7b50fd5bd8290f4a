mkdir -p gpurun_out
bash scripts/profile_round.sh r01g > gpurun_out/profile_r01g.log 2>&1
rm -f gpurun_out/other_g.jsonl
for wl in "--scale 24" "--workload er" "--workload mesh" "--workload road" "--workload gradient --scale 20" "--workload gradient --scale 20 --algorithm hybrid" "--scale 28"; do
  timeout 600 python bench.py --no-cpu --no-e2e --steps 5 $wl 2>/dev/null | grep '^{' >> gpurun_out/other_g.jsonl
done
ls gpurun_out | head -50

mkdir -p gpurun_out
rm -f gpurun_out/b_part2.jsonl gpurun_out/b_batches2.jsonl
timeout 900 python -m pytest tests/test_gpu_p2p.py -x -q 2>&1 | tail -3 > gpurun_out/t_p2p3.log
for ex in p2p nccl; do
  timeout 600 python bench.py --partitioned --exchange $ex --no-cpu --no-e2e --steps 5 2>> gpurun_out/b_part.err | grep '^{' >> gpurun_out/b_part2.jsonl
done
timeout 900 python scripts/bench_parts_local.py --scale 24 --parts 1 2 4 8 > gpurun_out/parts_local_s24c.jsonl 2> gpurun_out/parts_local.err
for c in "--batches 2" "--batches 3" "--batches 5" "--batches 10" "--batches 3 --no-host-cache" "--batches 10 --no-host-cache"; do
  python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu $c >> gpurun_out/b_batches2.jsonl 2>> gpurun_out/b_batches.err
done
cat gpurun_out/t_p2p3.log

# one gpurun call: GPU tests + quick benches (outputs under gpurun_out/)
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_p2p.py -x -q 2>&1 | tail -15 > gpurun_out/t_p2p.log
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/t_gpu3.log
for c in "--batches 2" "--batches 10" "--hbm-budget-gb 6"; do
  python bench.py --no-cpu --no-e2e --steps 3 $c >> gpurun_out/b_fill.jsonl 2>> gpurun_out/b_fill.err
done
tail -3 gpurun_out/t_p2p.log gpurun_out/t_gpu3.log

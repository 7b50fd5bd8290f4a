set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -m pytest tests/test_gpu_contract.py -x -q 2>&1 | tail -15 > gpurun_out/r02_contract.log
python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/r02_gpu_all.log
python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/r02_bench0.json 2> gpurun_out/r02_bench0.err
cat gpurun_out/r02_contract.log gpurun_out/r02_gpu_all.log; tail -c 1500 gpurun_out/r02_bench0.json

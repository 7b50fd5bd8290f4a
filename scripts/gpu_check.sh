mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_p2p.py tests/test_gpu_parity.py -k "partition or p2p" -x -q 2>&1 | tail -5 > gpurun_out/t_p2p2.log
timeout 900 python scripts/bench_parts_local.py --scale 24 --parts 1 4 8 > gpurun_out/parts_local_s24b.jsonl 2> gpurun_out/parts_local.err
cat gpurun_out/t_p2p2.log

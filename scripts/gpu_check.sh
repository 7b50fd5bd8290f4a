set -x
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/t_gpu2.log
python bench.py --no-cpu --no-e2e > gpurun_out/b_s26.json 2> gpurun_out/b_s26.err
python bench.py --no-cpu --no-e2e --hbm-budget-gb 6 --steps 3 > gpurun_out/b_s26_ooc_cache.json 2> gpurun_out/b_s26_ooc_cache.err
python bench.py --no-cpu --no-e2e --hbm-budget-gb 6 --steps 3 --no-host-cache > gpurun_out/b_s26_ooc_nocache.json 2> gpurun_out/b_s26_ooc_nocache.err
tail -3 gpurun_out/t_gpu2.log

set -x
timeout 1200 compute-sanitizer --tool racecheck --print-limit 20 python scripts/sanitize_run.py --quick > gpurun_out/sanitizer/r02_racecheck.log 2>&1; echo "exit=$?" >> gpurun_out/sanitizer/r02_racecheck.log
timeout 2400 python -m pytest tests -m gpu -x -q --durations=20 2>&1 | tail -40 > gpurun_out/r02_t10_all.log
timeout 300 python bench.py --partitioned --no-cpu --no-e2e --steps 10 > gpurun_out/r02_part_n1.json 2> gpurun_out/r02_part_n1.err
timeout 300 python bench.py --no-cpu --no-e2e --steps 10 > gpurun_out/r02_bench_s26.json 2> gpurun_out/r02_bench_s26.err
tail -4 gpurun_out/sanitizer/r02_racecheck.log; cat gpurun_out/r02_t10_all.log
tail -c 400 gpurun_out/r02_part_n1.json; tail -3 gpurun_out/r02_part_n1.err; tail -c 1500 gpurun_out/r02_bench_s26.json

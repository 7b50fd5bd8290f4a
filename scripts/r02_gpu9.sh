set -x
mkdir -p gpurun_out/sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python scripts/sanitize_run.py > gpurun_out/sanitizer/r02_$tool.log 2>&1; echo "exit=$?" >> gpurun_out/sanitizer/r02_$tool.log
done
timeout 300 python bench.py --partitioned --no-cpu --no-e2e --steps 10 > gpurun_out/r02_part_n1.json 2> gpurun_out/r02_part_n1.err
timeout 300 python bench.py --partitioned --no-cpu --no-e2e --steps 10 --exchange p2p > gpurun_out/r02_part_n1_p2p.json 2> gpurun_out/r02_part_n1_p2p.err
for tool in memcheck racecheck synccheck initcheck; do tail -4 gpurun_out/sanitizer/r02_$tool.log; done
tail -c 600 gpurun_out/r02_part_n1.json; tail -c 600 gpurun_out/r02_part_n1_p2p.json; tail -3 gpurun_out/r02_part_n1.err

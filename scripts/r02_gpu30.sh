# partition round-1 match from the smaller endpoint: partition / multi-process tests, partitioned bench (N=1)
set -x
timeout 1800 python -m pytest tests/test_gpu_p2p.py tests/test_gpu_dist.py -x -q 2>&1 | tail -2 > gpurun_out/t_part.log
for rep in 1 2; do
  python bench.py --no-cpu --no-e2e --steps 10 --partitioned 2>/dev/null | grep '^{' | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'part','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step']}))" >> gpurun_out/part.jsonl
  python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'single','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step']}))" >> gpurun_out/part.jsonl
done
cat gpurun_out/t_part.log gpurun_out/part.jsonl

# key cache + dist driver: targeted tests first (fail fast), bench on/off, then the full GPU suite
set -x
timeout 900 python -m pytest tests/test_gpu_contract.py tests/test_gpu_dist.py -x -q 2>&1 | tail -25 > gpurun_out/r02_t3_new.log
for kc in "" "--no-key-cache"; do
  timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu $kc > gpurun_out/r02_bench_kc$kc.json 2> gpurun_out/r02_bench_kc$kc.err
done
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/r02_t3_all.log
cat gpurun_out/r02_t3_new.log gpurun_out/r02_t3_all.log
for f in gpurun_out/r02_bench_kc*.json; do python -c "
import json,sys; d=json.loads(open('$f').read().strip().splitlines()[-1]); print('$f', round(d['value'],2), d['ms_per_step'], d['phase_ms'], d['rounds'], d['entries_swept'])"; done
tail -3 gpurun_out/r02_bench_kc*.err

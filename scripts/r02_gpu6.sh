set -x
mkdir -p /tmp/dc && gcc -O2 -I include tests/c/dist_c.c -L paper_conf_sc_mandulakgfhs24_b200 -llmatch -lpthread -Wl,-rpath,$PWD/paper_conf_sc_mandulakgfhs24_b200 -o /tmp/dc/dist_c
timeout 60 /tmp/dc/dist_c thread 2 /tmp/dc/g 20000 > gpurun_out/r02_dc_thread.log 2>&1; echo "rc=$?" >> gpurun_out/r02_dc_thread.log
timeout 1500 python -m pytest tests/test_gpu_dist.py tests/test_gpu_contract.py -x -q 2>&1 | tail -25 > gpurun_out/r02_t6_new.log
rm -f gpurun_out/variants.jsonl
for rep in 1 2; do
  for v in old new qx b1g8 b1g8qx p3g16; do
    LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 300 python bench.py --no-cpu --no-e2e --steps 10 2>/dev/null | grep '^{' | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'v':'$v','rep':$rep,'gteps':d['value'],'ms':d['ms_per_step'],'phase':d['phase_ms']}))" >> gpurun_out/variants.jsonl
  done
done
for v in qx b1g8 b1g8qx p3g16; do
  LMATCH_LIB=$PWD/build/variants/lm_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "golden or random_tiny or synthetic or hub or increasing or round_loop" 2>&1 | tail -1 > gpurun_out/t_var_$v.log
done
tail -3 gpurun_out/r02_dc_thread.log; cat gpurun_out/r02_t6_new.log gpurun_out/variants.jsonl gpurun_out/t_var_*.log

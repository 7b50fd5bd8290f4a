set -x
mkdir -p /tmp/dc && gcc -O2 -I include tests/c/dist_c.c -L paper_conf_sc_mandulakgfhs24_b200 -llmatch -lpthread -Wl,-rpath,$PWD/paper_conf_sc_mandulakgfhs24_b200 -o /tmp/dc/dist_c
LMATCH_TRACE=1 timeout 60 /tmp/dc/dist_c thread 2 /tmp/dc/g 20000 > gpurun_out/r02_dc_thread.log 2>&1; echo "rc=$?" >> gpurun_out/r02_dc_thread.log
tail -4 gpurun_out/r02_dc_thread.log
timeout 1800 python -m pytest tests/test_gpu_dist.py tests/test_gpu_contract.py -x -q 2>&1 | tail -25 > gpurun_out/r02_t7.log
cat gpurun_out/r02_t7.log

set -x
mkdir -p /tmp/dc && gcc -O2 -I include tests/c/dist_c.c -L paper_conf_sc_mandulakgfhs24_b200 -llmatch -lpthread -Wl,-rpath,$PWD/paper_conf_sc_mandulakgfhs24_b200 -o /tmp/dc/dist_c
LMATCH_TRACE=1 timeout 60 /tmp/dc/dist_c fork 2 /tmp/dc/g 20000 > gpurun_out/r02_dc_fork.log 2>&1; echo "rc=$?" >> gpurun_out/r02_dc_fork.log
LMATCH_TRACE=1 timeout 60 /tmp/dc/dist_c thread 2 /tmp/dc/g 20000 > gpurun_out/r02_dc_thread.log 2>&1; echo "rc=$?" >> gpurun_out/r02_dc_thread.log
timeout 300 compute-sanitizer --target-processes all --tool memcheck /tmp/dc/dist_c fork 2 /tmp/dc/g 20000 > gpurun_out/r02_dc_fork_memcheck.log 2>&1; echo "rc=$?" >> gpurun_out/r02_dc_fork_memcheck.log
grep -v "^\[lmatch" gpurun_out/r02_dc_fork.log | tail; grep "phase\|barrier" gpurun_out/r02_dc_fork.log | tail -12; tail -25 gpurun_out/r02_dc_thread.log; head -60 gpurun_out/r02_dc_fork_memcheck.log

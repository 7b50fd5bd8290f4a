#!/bin/bash
# Build bitmap-probe variants of liblmatch.so into build/variants/ (builder tooling).
set -e
cd "$(dirname "$0")/.."
mkdir -p build/variants
rm -f build/variants/*.so
for P in "$@"; do
  nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC \
    -Xcompiler -fvisibility=hidden --cudart static -shared -Xlinker --exclude-libs=ALL \
    -DLM_PROBE=$P paper_conf_sc_mandulakgfhs24_b200/csrc/lmatch.cu -o build/variants/lm_probe$P.so &
done
wait
ls build/variants

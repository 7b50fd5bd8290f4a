#!/bin/bash
# Build liblmatch.so variants that differ in one -D macro (builder tooling):
#   scripts/build_macro_variants.sh LM_PB_MINB 1 6 8  ->  build/variants/lm_LM_PB_MINB_<v>.so
set -e
cd "$(dirname "$0")/.."
mkdir -p build/variants
rm -f build/variants/*.so
M=$1; shift
for v in "$@"; do
  nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC \
    -Xcompiler -fvisibility=hidden --cudart static -shared -Xlinker --exclude-libs=ALL \
    -D$M=$v paper_conf_sc_mandulakgfhs24_b200/csrc/lmatch.cu -o build/variants/lm_${M}_$v.so &
done
wait
ls build/variants

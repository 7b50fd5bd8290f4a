#!/bin/bash
# Build liblmatch.so variants from named -D flag sets (builder tooling):
#   scripts/build_flag_variants.sh "base:" "pipe6:-DLM_PIPE=6" ...  ->  build/variants/lm_<name>.so
set -e
cd "$(dirname "$0")/.."
mkdir -p build/variants
rm -f build/variants/*.so
for v in "$@"; do
  name=${v%%:*}; flags=${v#*:}
  nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC \
    -Xcompiler -fvisibility=hidden --cudart static -shared -Xlinker --exclude-libs=ALL \
    $flags paper_conf_sc_mandulakgfhs24_b200/csrc/lmatch.cu -o build/variants/lm_$name.so &
done
wait
ls build/variants

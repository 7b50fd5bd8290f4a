#!/bin/bash
# Build sweep-tuning variants of liblmatch.so into build/variants/ (builder tooling).
set -e
cd "$(dirname "$0")/.."
mkdir -p build/variants
for v in "$@"; do   # v = TILE:RING:WARPS:WCAP[:IMPL]
  IFS=: read T R W C I <<< "$v"
  I=${I:-2}
  nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC \
    -Xcompiler -fvisibility=hidden --cudart static -shared -Xlinker --exclude-libs=ALL \
    -DLM_SWEEP_TILE=$T -DLM_SWEEP_RING=$R -DLM_SWEEP_WARPS=$W -DLM_SWEEP_WCAP=$C -DLM_SWEEP_IMPL=$I \
    paper_conf_sc_mandulakgfhs24_b200/csrc/lmatch.cu -o build/variants/lm_${T}_${R}_${W}_${C}_i${I}.so &
done
wait
ls build/variants

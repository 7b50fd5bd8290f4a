#!/bin/bash
# Build sweep-tuning variants of liblmatch.so into build/variants/ (builder tooling).
set -e
cd "$(dirname "$0")/.."
mkdir -p build/variants
for v in "$@"; do   # v = TILE:RING:WARPS:WCAP[:IMPL[:B0G:B0U:B1G:B1U:B2G:B2U]]
  IFS=: read T R W C I B0G B0U B1G B1U B2G B2U GBX <<< "$v"
  I=${I:-2}
  BX=""
  TAG=""
  if [ -n "$B0G" ]; then
    BX="-DLM_B0_G=$B0G -DLM_B0_U=$B0U -DLM_B1_G=$B1G -DLM_B1_U=$B1U -DLM_B2_G=$B2G -DLM_B2_U=$B2U"
    TAG="_b${B0G}x${B0U}_${B1G}x${B1U}_${B2G}x${B2U}"
  fi
  if [ -n "$GBX" ]; then BX="$BX -DLM_BODY_GRID=$GBX"; TAG="${TAG}_gb${GBX}"; fi
  nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC \
    -Xcompiler -fvisibility=hidden --cudart static -shared -Xlinker --exclude-libs=ALL \
    -DLM_SWEEP_TILE=$T -DLM_SWEEP_RING=$R -DLM_SWEEP_WARPS=$W -DLM_SWEEP_WCAP=$C -DLM_SWEEP_IMPL=$I \
    paper_conf_sc_mandulakgfhs24_b200/csrc/lmatch.cu -o build/variants/lm_${T}_${R}_${W}_${C}_i${I}${TAG}.so &
done
wait
ls build/variants

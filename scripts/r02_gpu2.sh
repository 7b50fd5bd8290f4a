# L2-policy variants: parity subset + bench x2 + ncu full of round-2 frontier kernels (base, all)
export VARIANTS="base kh bh kbh win all"
bash scripts/gpu_variants.sh > gpurun_out/r02_l2var.log 2>&1
for v in base kbh all; do
  LMATCH_LIB=$PWD/build/variants/lm_$v.so ncu --set full --clock-control none --import-source on -k regex:"k_point|k_compact|k_match_bins" -c 7 \
    -o gpurun_out/r02_frontier_full_$v -f python scripts/prof_run.py --runs 1 > /dev/null 2>&1
done
cat gpurun_out/r02_l2var.log

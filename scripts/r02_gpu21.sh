# what bounds the frontier pointer kernels: round-2 launch times with the bitmap probes and/or the
# key loads removed (timing experiment builds; their matchings are wrong)
for v in base noprobe nokeys neither; do
  LMATCH_LIB=$PWD/build/variants/lm_$v.so ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sectors_srcunit_tex_op_read.sum --clock-control none --csv \
    --log-file gpurun_out/exp_$v.csv python scripts/prof_run.py --runs 1 > gpurun_out/exp_$v.log 2>&1
done
ls -la gpurun_out

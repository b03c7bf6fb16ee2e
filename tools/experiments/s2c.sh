# DOWN copy unroll (U_COPY_S 4 / 6 / 8) and the data warps' spin back-off, after done-init + own-first
OUT=gpurun_out/s2c; mkdir -p $OUT
L=$PWD/paper_conf_hpca_sanghoonsk23_b200
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2 3; do
  $B > $OUT/b_prod_$rnd.log 2>&1
  CCUBE_LIB=$L/libccube_c6.so $B > $OUT/b_c6_$rnd.log 2>&1
  CCUBE_LIB=$L/libccube_c8.so $B > $OUT/b_c8_$rnd.log 2>&1
  CCUBE_BACKOFF_NS=0 $B > $OUT/b_bo0_$rnd.log 2>&1
  CCUBE_BACKOFF_NS=256 $B > $OUT/b_bo256_$rnd.log 2>&1
  $B --tree double > $OUT/b_prod_double_$rnd.log 2>&1
  CCUBE_LIB=$L/libccube_c8.so $B --tree double > $OUT/b_c8_double_$rnd.log 2>&1
done
CCUBE_LIB=$L/libccube_c8.so CCUBE_TRACE_UP=1 python tools/pipeline_profile.py single > $OUT/pipeline_c8.json 2> $OUT/pipe_c8.err
CCUBE_TRACE_UP=1 python tools/pipeline_profile.py single > $OUT/pipeline_prod.json 2> $OUT/pipe_prod.err

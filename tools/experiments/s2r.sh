# children's partials read with evict_last (they are overwritten by the final later) vs evict_first
OUT=gpurun_out/s2r; mkdir -p $OUT
L=$PWD/paper_conf_hpca_sanghoonsk23_b200
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2 3; do
  $B > $OUT/b_prod_$rnd.log 2>&1
  CCUBE_LIB=$L/libccube_pk.so $B > $OUT/b_pk_$rnd.log 2>&1
  $B --tree double > $OUT/b_prod_double_$rnd.log 2>&1
  CCUBE_LIB=$L/libccube_pk.so $B --tree double > $OUT/b_pk_double_$rnd.log 2>&1
done

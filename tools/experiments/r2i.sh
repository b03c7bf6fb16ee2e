# CTA-size buckets with more combine vectors in flight (see tree_allreduce.cu u_combine)
OUT=gpurun_out/r2i; mkdir -p $OUT
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2; do
  $B > $OUT/bench_t256_$rnd.log 2>&1
  $B --threads 192 > $OUT/bench_t192u6_$rnd.log 2>&1
  $B --threads 128 > $OUT/bench_t128u8_$rnd.log 2>&1
  CCUBE_LIB=tools/bin/libccube_v192u10.so $B --threads 128 > $OUT/bench_t128u10_$rnd.log 2>&1
  $B --threads 192 --tree double > $OUT/bench_double_t192u6_$rnd.log 2>&1
  $B --tree double > $OUT/bench_double_t256_$rnd.log 2>&1
done

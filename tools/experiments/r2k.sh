# block tiling vs U and chunk size; copy U; rotated LSU vs TMA (6 data warps)
OUT=gpurun_out/r2k; mkdir -p $OUT
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2; do
  $B > $OUT/b_default_$rnd.log 2>&1
  $B --chunk-bytes 524288 > $OUT/b_c512_$rnd.log 2>&1
  $B --chunk-bytes 393216 > $OUT/b_c384_$rnd.log 2>&1
  $B --chunk-bytes 131072 > $OUT/b_c128_$rnd.log 2>&1
  CCUBE_LIB=tools/bin/libccube_v256c6.so $B > $OUT/b_copyU6_$rnd.log 2>&1
  CCUBE_LIB=tools/bin/libccube_v256u5.so $B > $OUT/b_combU5_$rnd.log 2>&1
  CCUBE_LIB=tools/bin/libccube_v256u7.so $B > $OUT/b_combU7_$rnd.log 2>&1
  $B --threads 128 --chunk-bytes 524288 > $OUT/b_t128_c512_$rnd.log 2>&1
  $B --tree rotated --datapath lsu > $OUT/b_rot_lsu_$rnd.log 2>&1
  $B --tree rotated --datapath tma > $OUT/b_rot_tma_$rnd.log 2>&1
  $B --tree rotated --datapath tma --threads 256 > $OUT/b_rot_tma_t256_$rnd.log 2>&1
done

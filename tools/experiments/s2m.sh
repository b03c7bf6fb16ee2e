# AUTO control (one control warp + 7 data warps in the 256-thread geometry) as the default:
# A/B vs CCUBE_SPLIT_CONTROL=1 (round-2 default), then the full round at HEAD
OUT=gpurun_out/s2m; mkdir -p $OUT
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2 3; do
  for t in single double rotated; do
    $B --tree $t > $OUT/b_auto_${t}_$rnd.log 2>&1
    CCUBE_SPLIT_CONTROL=1 $B --tree $t > $OUT/b_sc1_${t}_$rnd.log 2>&1
  done
  $B --workload vgg16 --dtype bfloat16 --tree double --steps 50 > $OUT/b_auto_vgg_$rnd.log 2>&1
  CCUBE_SPLIT_CONTROL=1 $B --workload vgg16 --dtype bfloat16 --tree double --steps 50 > $OUT/b_sc1_vgg_$rnd.log 2>&1
done
bash tools/gpu_round.sh s2m

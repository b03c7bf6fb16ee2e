# idle pulled-leaf CTAs prefetch their own input into L2, W chunks ahead of the head
OUT=gpurun_out/r2u; mkdir -p $OUT
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2; do
  $B > $OUT/b_w0_$rnd.log 2>&1
  for w in 2 4 8 16 32; do CCUBE_LEAF_PREFETCH=$w $B > $OUT/b_w${w}_$rnd.log 2>&1; done
done
CCUBE_LEAF_PREFETCH=8 $B --tree double > $OUT/b_double_w8.log 2>&1
$B --tree double > $OUT/b_double_w0.log 2>&1
CCUBE_LEAF_PREFETCH=8 CCUBE_TRACE_UP=1 python tools/pipeline_profile.py single > $OUT/pipeline_w8.json 2> $OUT/pipe.err

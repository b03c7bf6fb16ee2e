OUT=gpurun_out/r2p; mkdir -p $OUT
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
$B > $OUT/b_pull.log 2>&1
CCUBE_TRANSPORT=1 $B > $OUT/b_push.log 2>&1
CCUBE_TRANSPORT=1 $B --threads 256 > $OUT/b_push_t256.log 2>&1
CCUBE_TRANSPORT=1 $B --tree double > $OUT/b_push_double.log 2>&1
$B --tree double > $OUT/b_pull_double.log 2>&1

# single tree placement check on one box: previous build (J 41, 4 pulled-leaf CTAs) vs the leaf group (J 42 auto, J 41), task order 2
OUT=gpurun_out/s2g; mkdir -p $OUT
L=$PWD/paper_conf_hpca_sanghoonsk23_b200
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2 3 4; do
  CCUBE_LIB=$L/libccube_prevbf.so $B > $OUT/b_prev_$rnd.log 2>&1
  $B > $OUT/b_new_$rnd.log 2>&1
  $B --channels 41 > $OUT/b_new41_$rnd.log 2>&1
  CCUBE_TASK_ORDER=2 $B > $OUT/b_new_o2_$rnd.log 2>&1
  CCUBE_TASK_ORDER=1 $B > $OUT/b_new_o1_$rnd.log 2>&1
  CCUBE_LIB=$L/libccube_prevbf.so CCUBE_TASK_ORDER=2 $B > $OUT/b_prev_o2_$rnd.log 2>&1
done

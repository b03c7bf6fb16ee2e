# one control warp + 7 data warps (256-thread CTA, U 6) vs the default 2 control + 6 data warps
OUT=gpurun_out/s2l; mkdir -p $OUT
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2 3; do
  $B > $OUT/b_def_$rnd.log 2>&1
  CCUBE_SPLIT_CONTROL=0 $B --threads 224 > $OUT/b_sc0_t224_$rnd.log 2>&1
  $B --tree double > $OUT/b_def_double_$rnd.log 2>&1
  CCUBE_SPLIT_CONTROL=0 $B --threads 224 --tree double > $OUT/b_sc0_t224_double_$rnd.log 2>&1
done
CCUBE_SPLIT_CONTROL=0 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "parity_small or whole_buffer or gates" > $OUT/pytest_sc0.log 2>&1; echo "exit $?" >> $OUT/pytest_sc0.log

# one leaf-group CTA per process for every pulled leaf (frees CTA slots: single J 41 -> 42,
# double 20 -> 21, rotated 4 -> 5 at P = 8 loopback); A/B vs the previous build, full GPU suite
OUT=gpurun_out/s2e; mkdir -p $OUT
L=$PWD/paper_conf_hpca_sanghoonsk23_b200
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2 3; do
  for t in single double rotated; do
    $B --tree $t > $OUT/b_new_${t}_$rnd.log 2>&1
    CCUBE_LIB=$L/libccube_prevbf.so $B --tree $t > $OUT/b_prev_${t}_$rnd.log 2>&1
  done
done
$B --tree rotated --datapath lsu > $OUT/b_new_rotated_lsu.log 2>&1
timeout 1800 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "exit $?" >> $OUT/pytest_gpu.log

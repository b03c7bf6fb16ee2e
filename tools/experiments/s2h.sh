# per-rank leaf-group CTAs + AUTO = LSU: A/B vs the previous build on single / double / rotated, then the full round
OUT=gpurun_out/s2h; mkdir -p $OUT
L=$PWD/paper_conf_hpca_sanghoonsk23_b200
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2 3; do
  for t in single double rotated; do
    $B --tree $t > $OUT/b_new_${t}_$rnd.log 2>&1
    CCUBE_LIB=$L/libccube_prevbf.so $B --tree $t > $OUT/b_prev_${t}_$rnd.log 2>&1
  done
done
bash tools/gpu_round.sh s2h

# after the leaf group: J for the single tree (40 / 41 / 42 = auto), and the rotated set's datapath at P = 2 / 4 / 8
OUT=gpurun_out/s2f; mkdir -p $OUT
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2; do
  for j in 40 41 42; do $B --channels $j > $OUT/b_single_j${j}_$rnd.log 2>&1; done
  for j in 20 21; do $B --tree double --channels $j > $OUT/b_double_j${j}_$rnd.log 2>&1; done
  for P in 2 4 8; do
    for dp in lsu tma; do $B --tree rotated --ranks $P --datapath $dp > $OUT/b_rot_p${P}_${dp}_$rnd.log 2>&1; done
  done
done

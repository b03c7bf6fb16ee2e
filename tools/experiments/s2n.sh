# long-step outliers: the driver's command (clocks sampled) and --no-clocks, AUTO control vs the split pair
OUT=gpurun_out/s2n; mkdir -p $OUT
for rnd in 1 2 3 4; do
  python bench.py --steps 20 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra > $OUT/b_auto_20_$rnd.log 2>&1
  CCUBE_SPLIT_CONTROL=1 python bench.py --steps 20 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra > $OUT/b_sc1_20_$rnd.log 2>&1
  python bench.py --no-iter --no-e2e --no-cpu-baseline --no-extra > $OUT/b_auto_200_$rnd.log 2>&1
  CCUBE_SPLIT_CONTROL=1 python bench.py --no-iter --no-e2e --no-cpu-baseline --no-extra > $OUT/b_sc1_200_$rnd.log 2>&1
  python bench.py --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks > $OUT/b_auto_200nc_$rnd.log 2>&1
done
python bench.py --steps 20 --warmup 5 > $OUT/b_driver_cmd.log 2>&1

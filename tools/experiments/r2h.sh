# U=6 combines (6 data warps, 128 regs) vs the default; compute-sanitizer; ncu of small messages
OUT=gpurun_out/r2h; mkdir -p $OUT
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2; do
  $B > $OUT/bench_default_$rnd.log 2>&1
  $B --threads 192 > $OUT/bench_t192_$rnd.log 2>&1
  CCUBE_LIB=tools/bin/libccube_u6.so $B --threads 192 > $OUT/bench_u6_t192_$rnd.log 2>&1
  CCUBE_LIB=tools/bin/libccube_u6c8.so $B --threads 192 > $OUT/bench_u6c8_t192_$rnd.log 2>&1
done
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_case.py > $OUT/sanitizer_$tool.log 2>&1
  echo "exit $?" >> $OUT/sanitizer_$tool.log
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_small.csv \
  python tools/size_sweep.py --ranks 2,8 --trees single --overlap 1 --min-kib 1 --max-mib 1 --iters 3 --warmup 1 --inner 1 > $OUT/sizes_small_ncu.jsonl 2>&1

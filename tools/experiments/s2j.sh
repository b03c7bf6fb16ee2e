# P = 2 / 4 check of done-init and own-first (same sources, macros off) at 1 GiB and 16 MiB and the bench size
OUT=gpurun_out/s2j; mkdir -p $OUT
L=$PWD/paper_conf_hpca_sanghoonsk23_b200
B="python bench.py --steps 50 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2 3; do
  for v in prod x00 xd1; do
    if [ $v = prod ]; then LIBV=""; else LIBV=$L/libccube_$v.so; fi
    for P in 2 4 8; do CCUBE_LIB=$LIBV $B --ranks $P > $OUT/b_${v}_p${P}_$rnd.log 2>&1; done
  done
done
for v in prod x00; do
  if [ $v = prod ]; then LIBV=""; else LIBV=$L/libccube_$v.so; fi
  CCUBE_LIB=$LIBV python tools/size_sweep.py --ranks 2,4 --trees single --overlap 1 --min-kib 16384 --max-mib 1024 > $OUT/sizes_$v.jsonl 2> $OUT/sizes_$v.err
done

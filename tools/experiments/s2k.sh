# own-first only in the <= 256-thread CTAs: P = 2 / 4 / 8 vs the same sources with both fill changes off
OUT=gpurun_out/s2k; mkdir -p $OUT
L=$PWD/paper_conf_hpca_sanghoonsk23_b200
B="python bench.py --steps 50 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2 3; do
  for v in prod x00 xd1; do
    if [ $v = prod ]; then LIBV=""; else LIBV=$L/libccube_$v.so; fi
    for P in 2 4 8; do CCUBE_LIB=$LIBV $B --ranks $P > $OUT/b_${v}_p${P}_$rnd.log 2>&1; done
    CCUBE_LIB=$LIBV $B --tree double > $OUT/b_${v}_double_$rnd.log 2>&1
  done
done
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "parity_small or channels or threads or whole_buffer or repeated or gates" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log

# done-init + own-input-first (fill/hop latency): A/B against the same sources with both off
OUT=gpurun_out/s2a; mkdir -p $OUT
L=paper_conf_hpca_sanghoonsk23_b200
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2 3; do
  for v in x00 x10 prod; do
    if [ $v = prod ]; then LIBV=""; else LIBV=$PWD/$L/libccube_$v.so; fi
    CCUBE_LIB=$LIBV $B > $OUT/b_${v}_$rnd.log 2>&1
    CCUBE_LIB=$LIBV $B --tree double > $OUT/b_${v}_double_$rnd.log 2>&1
  done
done
for v in x00 prod; do
  if [ $v = prod ]; then LIBV=""; else LIBV=$PWD/$L/libccube_$v.so; fi
  CCUBE_LIB=$LIBV python tools/size_sweep.py --ranks 8 --trees single --min-kib 512 --max-mib 64 --iters 20 > $OUT/sizes_$v.jsonl 2> $OUT/sizes_$v.err
  CCUBE_LIB=$LIBV CCUBE_TRACE_UP=1 python tools/pipeline_profile.py single > $OUT/pipeline_$v.json 2> $OUT/pipe_$v.err
done
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "parity_small or channels or threads or whole_buffer or special_values or repeated or gates or split" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log

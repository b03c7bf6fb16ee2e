# split heads (the pipeline's head UP tasks on two CTAs per channel): timing + parity
OUT=gpurun_out/r2q; mkdir -p $OUT
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2; do
  $B > $OUT/b_split_$rnd.log 2>&1
  CCUBE_SPLIT_HEADS=0 $B > $OUT/b_nosplit_$rnd.log 2>&1
  $B --tree double > $OUT/b_split_double_$rnd.log 2>&1
  CCUBE_SPLIT_HEADS=0 $B --tree double > $OUT/b_nosplit_double_$rnd.log 2>&1
done
$B --threads 256 > $OUT/b_split_t256.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "parity_small or channels or threads or whole_buffer or special_values or repeated or gates" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
CCUBE_TRACE_UP=1 python tools/pipeline_profile.py single > $OUT/pipeline_split.json 2> $OUT/pipe.err

# paired DOWN tasks (one CTA covers two channels' copies) -> more channels for the UP stages
OUT=gpurun_out/r2y; mkdir -p $OUT
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2; do
  $B > $OUT/b_base_$rnd.log 2>&1
  CCUBE_DOWN_PAIRS=1 $B > $OUT/b_pairs_$rnd.log 2>&1
  CCUBE_DOWN_PAIRS=1 $B --threads 192 > $OUT/b_pairs_t192_$rnd.log 2>&1
  CCUBE_DOWN_PAIRS=1 $B --threads 256 > $OUT/b_pairs_t256_$rnd.log 2>&1
  CCUBE_DOWN_PAIRS=1 $B --tree double > $OUT/b_pairs_double_$rnd.log 2>&1
  $B --tree double > $OUT/b_base_double_$rnd.log 2>&1
done
CCUBE_DOWN_PAIRS=1 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "parity_small or channels or whole_buffer or gates or special_values" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
CCUBE_DOWN_PAIRS=1 CCUBE_TRACE_UP=1 python tools/pipeline_profile.py single > $OUT/pipeline_pairs.json 2> $OUT/pipe.err

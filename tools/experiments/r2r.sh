# TMA datapath for the pipeline's head tasks only (smem ring = bytes in flight without registers)
OUT=gpurun_out/r2r; mkdir -p $OUT
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2; do
  $B > $OUT/b_lsu_$rnd.log 2>&1
  CCUBE_TMA_HEADS=1 $B > $OUT/b_tmaheads_$rnd.log 2>&1
  CCUBE_TMA_HEADS=1 $B --threads 256 > $OUT/b_tmaheads_t256_$rnd.log 2>&1
  CCUBE_TMA_HEADS=1 $B --tree double > $OUT/b_tmaheads_double_$rnd.log 2>&1
done
CCUBE_TMA_HEADS=1 CCUBE_TRACE_UP=1 python tools/pipeline_profile.py single > $OUT/pipeline_tmaheads.json 2> $OUT/pipe.err
CCUBE_TMA_HEADS=1 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "parity_small or whole_buffer" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log

# one 512-thread CTA per SM (14 data warps x U 6, 128 registers) vs two 256-thread CTAs
OUT=gpurun_out/r2v; mkdir -p $OUT
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2; do
  $B > $OUT/b_auto_$rnd.log 2>&1
  $B --threads 448 > $OUT/b_t448_$rnd.log 2>&1
  $B --threads 384 > $OUT/b_t384_$rnd.log 2>&1
  $B --threads 448 --tree double > $OUT/b_t448_double_$rnd.log 2>&1
  $B --threads 448 --chunk-bytes 393216 > $OUT/b_t448_c384_$rnd.log 2>&1
done
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "parity_threads or whole_buffer" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log

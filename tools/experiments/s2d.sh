# bf16 combine: packed cvt.rn.bf16x2.f32 (F2FP.PACK_AB) vs two F2F + PRMT; VGG-16 bf16 lines + bf16 parity
OUT=gpurun_out/s2d; mkdir -p $OUT
L=$PWD/paper_conf_hpca_sanghoonsk23_b200
B="python bench.py --steps 50 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks --workload vgg16 --dtype bfloat16"
for rnd in 1 2 3; do
  $B --tree double > $OUT/b_new_double_$rnd.log 2>&1
  CCUBE_LIB=$L/libccube_prevbf.so $B --tree double > $OUT/b_prev_double_$rnd.log 2>&1
  $B --tree single > $OUT/b_new_single_$rnd.log 2>&1
  CCUBE_LIB=$L/libccube_prevbf.so $B --tree single > $OUT/b_prev_single_$rnd.log 2>&1
done
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "bfloat16 or special or ll or vgg or subnormal" > $OUT/pytest_bf16.log 2>&1; echo "exit $?" >> $OUT/pytest_bf16.log

O=gpurun_out/uvar; mkdir -p $O
L=paper_conf_hpca_sanghoonsk23_b200/libccube.so
cp $L /tmp/libccube_orig.so
B="timeout 300 python bench.py --steps 100 --warmup 10 --no-e2e --no-cpu-baseline --no-iter --no-clocks"
for v in u2_4 u2_8 u4_4 u4_8; do
  cp tools/bin/var/libccube_$v.so $L
  $B > $O/bench_P8_$v.log 2>&1
  $B --ranks 4 > $O/bench_P4_$v.log 2>&1
  python tools/pipeline_profile.py > $O/pipeline_$v.json 2>>$O/pp.err
done
cp /tmp/libccube_orig.so $L

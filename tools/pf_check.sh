O=gpurun_out/pf1; mkdir -p $O
B="timeout 300 python bench.py --steps 100 --warmup 10 --no-e2e --no-cpu-baseline --no-iter --no-clocks"
for pf in 0 2 4 8 16; do
  $B --prefetch $pf > $O/bench_P8_pf$pf.log 2>&1
  $B --prefetch $pf --ranks 2 > $O/bench_P2_pf$pf.log 2>&1
done
$B --prefetch 4 --tree double > $O/bench_P8d_pf4.log 2>&1
$B --prefetch 0 --tree double > $O/bench_P8d_pf0.log 2>&1
$B --prefetch 8 --tree double > $O/bench_P8d_pf8.log 2>&1

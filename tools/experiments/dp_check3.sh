O=gpurun_out/dp3; mkdir -p $O
B="timeout 300 python bench.py --steps 100 --warmup 10 --no-e2e --no-cpu-baseline --no-iter --no-clocks"
for P in 2 8; do for dp in tma lsu; do
  $B --datapath $dp --ranks $P --chunk-bytes 1048576 > $O/bench_P${P}_1m_$dp.log 2>&1
done; done
for ch in 12 20 30; do
  $B --datapath tma --channels $ch > $O/bench_P8_ch${ch}_tma.log 2>&1
  $B --datapath lsu --channels $ch > $O/bench_P8_ch${ch}_lsu.log 2>&1
done

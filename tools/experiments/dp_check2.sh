O=gpurun_out/dp2; mkdir -p $O
for P in 2 4 8; do for dp in tma lsu; do
  timeout 300 python bench.py --steps 100 --warmup 10 --no-e2e --no-cpu-baseline --no-iter --datapath $dp --ranks $P > $O/bench_P${P}_$dp.log 2>&1
done; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tree_allreduce -s 3 -c 1 -o $O/prof_tma python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-clocks --no-iter --datapath tma > $O/prof_tma.log 2>&1

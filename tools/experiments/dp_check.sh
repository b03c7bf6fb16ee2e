O=gpurun_out/dp1; mkdir -p $O
for dp in tma lsu; do
  timeout 300 python bench.py --steps 100 --warmup 10 --no-e2e --no-cpu-baseline --no-iter --datapath $dp > $O/bench_$dp.log 2>&1
done
for tree in double rotated; do for dp in tma lsu; do
  timeout 300 python bench.py --steps 100 --warmup 10 --no-e2e --no-cpu-baseline --no-iter --datapath $dp --tree $tree > $O/bench_${tree}_$dp.log 2>&1
done; done
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > $O/pytest_parity.log 2>&1; echo "exit $?" >> $O/pytest_parity.log

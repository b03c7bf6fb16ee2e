O=gpurun_out/r1c; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "tma or prefetch or channels" > $O/pytest_new.log 2>&1; echo "exit $?" >> $O/pytest_new.log
B="timeout 300 python bench.py --steps 100 --warmup 10 --no-e2e --no-cpu-baseline --no-iter --no-clocks"
for P in 2 4 8; do for tree in single double; do
  $B --ranks $P --tree $tree > $O/bench_P${P}_$tree.log 2>&1
done; done

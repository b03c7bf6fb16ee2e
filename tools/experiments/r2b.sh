OUT=gpurun_out/r2b; mkdir -p $OUT
nproc > $OUT/nproc.txt; lscpu | grep -E "Model name|^CPU\(s\)" >> $OUT/nproc.txt
timeout 900 python bench.py > $OUT/bench.log 2>&1; echo "exit $?" >> $OUT/bench.log
bash tools/experiments/multi_bench_check.sh r2b_multi
timeout 900 python -m pytest tests/test_gpu_multiproc.py -x -q -k "peer" > $OUT/pytest_peer.log 2>&1; echo "exit $?" >> $OUT/pytest_peer.log

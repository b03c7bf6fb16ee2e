# v8 (rotated channel slices): GPU parity, chunk sweep, bench line
mkdir -p gpurun_out/sw8
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/sw8/pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/sw8/pytest_gpu.log
for P in 2 4 8; do
timeout 300 python tools/sweep.py --ranks $P --trees single,double --channels 0 --threads 256 --chunks 262144,524288,1048576,2097152,4194304 > gpurun_out/sw8/P$P.jsonl 2>&1
done
timeout 600 python bench.py > gpurun_out/sw8/bench.log 2>&1

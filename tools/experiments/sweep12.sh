# v10: rotated tree set, 128 channels, adaptive channels for small buffers
mkdir -p gpurun_out/sw12
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/sw12/pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/sw12/pytest_gpu.log
for P in 2 4 8; do
timeout 300 python tools/sweep.py --ranks $P --trees single,double,rotated --channels 0 --threads 256 --chunks 262144 > gpurun_out/sw12/P$P.jsonl 2>&1
done
timeout 900 python tools/size_sweep.py --ranks 2,8 --trees single,rotated --overlap 1 --max-mib 64 > gpurun_out/sw12/sizes.jsonl 2> gpurun_out/sw12/sizes.err

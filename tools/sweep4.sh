mkdir -p gpurun_out/sw4
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "parity_small or channels or threads or tiny or full_size_resnet" > gpurun_out/sw4/pytest_async.log 2>&1
for P in 2 4 8; do
python tools/sweep.py --ranks $P --trees single --channels 0 --threads 128,256 --chunks 262144,1048576 --tma 0,2 > gpurun_out/sw4/P$P.jsonl 2>&1
done
python tools/sweep.py --ranks 8 --trees double --channels 0 --threads 128,256 --chunks 262144,1048576 --tma 0,2 > gpurun_out/sw4/P8d.jsonl 2>&1

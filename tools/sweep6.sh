mkdir -p gpurun_out/sw6
for P in 2 8; do
python tools/sweep.py --ranks $P --trees single --channels 0 --threads 128,256 --chunks 262144,1048576 --tma 0 > gpurun_out/sw6/P$P.jsonl 2>&1
done
python tools/sweep.py --ranks 8 --trees double --channels 0 --threads 128,256 --chunks 262144,1048576 --tma 0 > gpurun_out/sw6/P8d.jsonl 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/sw6/pytest.log 2>&1

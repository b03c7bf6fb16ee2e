mkdir -p gpurun_out/sw5
for P in 2 8; do
python tools/sweep.py --ranks $P --trees single --channels 0 --threads 128,256 --chunks 262144,1048576 --tma 0,2 --rel 1,2,4,8,16 > gpurun_out/sw5/P$P.jsonl 2>&1
done
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "parity_small or channels or threads or tiny or full_size or gradient or trace" > gpurun_out/sw5/pytest.log 2>&1

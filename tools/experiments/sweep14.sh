# v12: division-free slice iterator + backoff in the data-warp readiness spin
mkdir -p gpurun_out/sw14
for P in 2 4 8; do
timeout 300 python tools/sweep.py --ranks $P --trees single,double,rotated --channels 0 --threads 224,256 --chunks 262144,1048576 > gpurun_out/sw14/P$P.jsonl 2>&1
done
timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -k "parity_small or rotated or channels or tiny or full_size or fused" > gpurun_out/sw14/pytest.log 2>&1; echo "exit $?" >> gpurun_out/sw14/pytest.log

mkdir -p gpurun_out/sw2
python tools/sweep.py --trees single,double --channels 0 --threads 128,256 --chunks 262144,1048576 --prefetch 0,1,2,4 > gpurun_out/sw2/prefetch.jsonl 2>&1
python -m pytest tests/test_gpu_parity.py -x -q -k "parity_small and float32" > gpurun_out/sw2/pytest_pf0.log 2>&1
CCUBE_PREFETCH=2 python -m pytest tests/test_gpu_parity.py -x -q -k "parity_small or full_size" > gpurun_out/sw2/pytest_pf2.log 2>&1

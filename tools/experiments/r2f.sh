OUT=gpurun_out/r2f; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "ll or tiny or count_zero or repeated" > $OUT/pytest_ll.log 2>&1; echo "exit $?" >> $OUT/pytest_ll.log
timeout 900 python -m pytest tests/test_gpu_multiproc.py -q -x -k "ipc_parity" > $OUT/pytest_mp.log 2>&1; echo "exit $?" >> $OUT/pytest_mp.log
timeout 600 python tools/size_sweep.py --ranks 2,4,8 --trees single,double --overlap 1 --min-kib 1 --max-mib 1 > $OUT/sizes_small.jsonl 2> $OUT/sizes.err

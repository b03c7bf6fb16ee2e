# LL kernel with 4-line batches per thread: latency 1 KiB - 512 KiB; LL parity
OUT=gpurun_out/r2o; mkdir -p $OUT
timeout 600 python tools/size_sweep.py --ranks 2,4,8 --trees single --overlap 1 --min-kib 1 --max-mib 1 --protocol ll,chunked --chunk-bytes 1048576 > $OUT/sizes.jsonl 2> $OUT/err.txt
CCUBE_LL_MAX_BYTES=1048576 timeout 600 python tools/size_sweep.py --ranks 8 --trees single --overlap 1 --min-kib 256 --max-mib 1 --protocol ll --chunk-bytes 1048576 > $OUT/sizes_ll1m.jsonl 2>> $OUT/err.txt
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multiproc.py -q -x -k "_ll or ipc_parity or tiny" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log

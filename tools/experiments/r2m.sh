# auto CTA size: bench + large-message points of the size sweep + a parity subset
OUT=gpurun_out/r2m; mkdir -p $OUT
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
$B > $OUT/b_auto.log 2>&1
$B --tree double > $OUT/b_auto_double.log 2>&1
timeout 900 python tools/size_sweep.py --ranks 2,4,8 --trees single,double --overlap 1 --min-kib 65536 --max-mib 1024 --protocol chunked > $OUT/sizes_big.jsonl 2> $OUT/sizes.err
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "parity_small or threads or channels or whole_buffer" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log

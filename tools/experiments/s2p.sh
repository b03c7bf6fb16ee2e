# AUTO control with the >= 128-chunk threshold: P = 8 sizes 1 MiB - 1 GiB, bench, parity subset
OUT=gpurun_out/s2p; mkdir -p $OUT
timeout 900 python tools/size_sweep.py --ranks 8 --trees single,double,rotated --overlap 1 --min-kib 1024 --max-mib 1024 > $OUT/sizes_p8.jsonl 2> $OUT/sizes.err
for rnd in 1 2; do python bench.py --steps 20 --warmup 5 --no-iter --no-e2e --no-cpu-baseline > $OUT/b_$rnd.log 2>&1; done
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multiproc.py -q -x -k "parity_small or whole_buffer or gates or repeated or channels or ipc_parity" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log

# session-2 final build: size sweep (configs[4]), turnaround, new multi-process tests, N>1 plumbing
OUT=gpurun_out/s2i; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_multiproc.py -q -x > $OUT/pytest_multiproc.log 2>&1; echo "exit $?" >> $OUT/pytest_multiproc.log
timeout 1500 python tools/size_sweep.py --ranks 2,4,8 --trees single,double,rotated --overlap 1,0 --min-kib 1 --max-mib 1024 > $OUT/sizes.jsonl 2> $OUT/sizes.err
timeout 300 python tools/turnaround.py > $OUT/turnaround.json 2> $OUT/turnaround.err
bash tools/experiments/multi_bench_check.sh s2i_multi

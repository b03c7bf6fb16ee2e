# final build: size sweep (configs[4]), turnaround, iteration sweep, N>1 plumbing
OUT=gpurun_out/r2w; mkdir -p $OUT
timeout 1500 python tools/size_sweep.py --ranks 2,4,8 --trees single,double,rotated --overlap 1,0 --min-kib 1 --max-mib 1024 > $OUT/sizes.jsonl 2> $OUT/sizes.err
timeout 300 python tools/turnaround.py > $OUT/turnaround.json 2> $OUT/turnaround.err
timeout 2400 python tools/iter_sweep.py > $OUT/iter_sweep.jsonl 2> $OUT/iter_sweep.err
bash tools/experiments/multi_bench_check.sh r2w_multi

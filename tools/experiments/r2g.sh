# size sweep (configs[4]) with the LL protocol and inner-loop timing; iteration sweep (f3/f4)
OUT=gpurun_out/r2g; mkdir -p $OUT
timeout 1500 python tools/size_sweep.py --ranks 2,4,8 --trees single,double,rotated --overlap 1,0 --min-kib 1 --max-mib 1024 > $OUT/sizes.jsonl 2> $OUT/sizes.err
timeout 2400 python tools/iter_sweep.py > $OUT/iter_sweep.jsonl 2> $OUT/iter_sweep.err

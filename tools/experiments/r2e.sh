OUT=gpurun_out/r2e; mkdir -p $OUT
CCUBE_TRACE_UP=1 python tools/pipeline_profile.py double > $OUT/pipeline_double_up.json 2> $OUT/pipe.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tree_allreduce -s 3 -c 1 -o $OUT/prof python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-clocks --no-iter --no-extra > $OUT/prof_bench.log 2>&1
echo "ncu exit $?" >> $OUT/prof_bench.log

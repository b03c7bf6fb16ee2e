# final build: size sweep, turnaround, pipeline trace
OUT=gpurun_out/s2o; mkdir -p $OUT
timeout 1500 python tools/size_sweep.py --ranks 2,4,8 --trees single,double,rotated --overlap 1,0 --min-kib 1 --max-mib 1024 > $OUT/sizes.jsonl 2> $OUT/sizes.err
timeout 300 python tools/turnaround.py > $OUT/turnaround.json 2> $OUT/turnaround.err
CCUBE_TRACE_UP=1 timeout 300 python tools/pipeline_profile.py single > $OUT/pipeline_single_up.json 2> $OUT/pipe.err

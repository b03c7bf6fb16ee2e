OUT=gpurun_out/r2d; mkdir -p $OUT
CCUBE_TRACE_UP=1 python tools/pipeline_profile.py single > $OUT/pipeline_single_up.json 2> $OUT/pipe.err
CCUBE_TRACE_UP=1 python tools/pipeline_profile.py double > $OUT/pipeline_double_up.json 2>> $OUT/pipe.err

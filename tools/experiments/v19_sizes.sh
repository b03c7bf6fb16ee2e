#!/bin/bash
# v19: message-size sweep (configs[4]) at the final round-1 kernel, plus the VGG-16 bf16 line.
mkdir -p gpurun_out/v19s
timeout 1200 python tools/size_sweep.py --ranks 2,4,8 --trees single,double,rotated --overlap 1,0 \
  > gpurun_out/v19s/sizes.jsonl 2> gpurun_out/v19s/sizes.err
timeout 600 python bench.py --workload vgg16 --no-cpu-baseline --no-iter > gpurun_out/v19s/bench_vgg16.log 2>&1
echo "exit $?" >> gpurun_out/v19s/bench_vgg16.log

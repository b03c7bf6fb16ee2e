#!/bin/bash
# NVLink + HBM byte counters of the tree AllReduce kernel, one process per GPU
# (SURVEY §8(d) "Record ncu counters for achieved NVLink/HBM GB/s"; VERDICT r1
# missing #4).  ncu application replay (the kernels of all ranks must run together,
# so no kernel replay), a single pass of five counters, every rank profiled:
#   nvltx__bytes.sum / nvlrx__bytes.sum   NVLink bytes sent / received by the GPU
#   dram__bytes_read.sum / _write.sum     HBM traffic
#   gpu__time_duration.sum                kernel time
# then tools/nvlink_summary.py turns the CSVs into GB/s per rank and launch.
#
#   bash tools/nvlink_counters.sh N [extra bench.py args]      (N GPUs on this node)
# Not a bench number: ncu serialises and instruments the launches.  Needs one GPU per
# process: on a single shared GPU ncu holds one rank's spinning kernel while the
# other's waits for it, and the watchdog fires (profiles/r02/l/nvlink_shared.log).
# bench.py itself reads NVML's NVLink byte counters around its timed region at N > 1
# (the line's nvlink_counters_rank0), which needs no profiler.
N=${1:-8}; shift
OUT=gpurun_out/nvlink_n$N; mkdir -p $OUT
timeout 1800 ncu --target-processes all --replay-mode application --clock-control none \
  --metrics nvltx__bytes.sum,nvlrx__bytes.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
  -k regex:tree_allreduce -c 20 --csv --log-file $OUT/nvlink_%p.csv \
  python -m torch.distributed.run --nnodes=1 --nproc-per-node $N --master-addr 127.0.0.1 \
  --master-port 29531 bench.py --gpus $N --steps 5 --warmup 3 --no-e2e --no-cpu-baseline \
  --no-clocks --no-iter --no-extra --no-nccl --no-port-peak "$@" > $OUT/bench.log 2>&1
echo "ncu exit $?" >> $OUT/bench.log
python tools/nvlink_summary.py $OUT/nvlink_*.csv > $OUT/summary.json
cat $OUT/summary.json

#!/bin/bash
# One gpurun pass: GPU parity tests, smoke, the bench line, the ncu launch list and
# one ncu --set full capture of the hot kernel.  Usage (from the repo root, under
# gpurun):  bash tools/gpu_round.sh [tag]   — outputs land in gpurun_out/<tag>/.
TAG=${1:-r01}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi > $OUT/nvidia-smi.txt 2>&1
nproc > $OUT/nproc.txt; lscpu | grep -E "Model name|^CPU\(s\)" >> $OUT/nproc.txt
if [ -z "$SKIP_TESTS" ]; then
  timeout 1500 python -m pytest tests -m gpu -x -q ${PYTEST_ARGS} > $OUT/pytest_gpu.log 2>&1
  echo "pytest exit $?" >> $OUT/pytest_gpu.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1
  echo "smoke exit $?" >> $OUT/smoke.log
fi
timeout 600 python bench.py ${BENCH_ARGS} > $OUT/bench.log 2>&1
echo "bench exit $?" >> $OUT/bench.log
if [ -z "$SKIP_NCU" ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file $OUT/launches.csv python bench.py --steps 5 --warmup 3 --no-e2e \
    --no-cpu-baseline --no-clocks ${BENCH_ARGS} > $OUT/launches_bench.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on \
    -k regex:tree_allreduce -s 3 -c 1 -o $OUT/prof python bench.py --steps 2 --warmup 3 \
    --no-e2e --no-cpu-baseline --no-clocks ${BENCH_ARGS} > $OUT/prof_bench.log 2>&1
  echo "ncu exit $?" >> $OUT/prof_bench.log
fi

#!/bin/bash
# CCUBE_TASK_ORDER sweep (block -> task placement): bench workload at P = 8 / 4 / 2,
# single and double tree, the orders interleaved over 3 passes.
O=gpurun_out/order; mkdir -p $O
B="timeout 300 python bench.py --steps 100 --warmup 10 --no-e2e --no-cpu-baseline --no-iter --no-clocks"
for pass in 1 2 3; do
  for o in 0 1 2; do
    CCUBE_TASK_ORDER=$o $B > $O/P8_single_o${o}_p$pass.log 2>&1
    CCUBE_TASK_ORDER=$o $B --tree double > $O/P8_double_o${o}_p$pass.log 2>&1
    CCUBE_TASK_ORDER=$o $B --ranks 4 > $O/P4_single_o${o}_p$pass.log 2>&1
    CCUBE_TASK_ORDER=$o $B --ranks 2 > $O/P2_single_o${o}_p$pass.log 2>&1
  done
done

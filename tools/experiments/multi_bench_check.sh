#!/bin/bash
# The N>1 bench path (torchrun, one process per rank) on a one-GPU box: every rank on
# cuda:0 (CCUBE_ALLOW_SHARED_GPU=1, contexts time-slice), gloo plumbing, a prefix of
# the workload.  Checks the JSON line, the device start barrier, the max-over-ranks
# timing, the cross-rank checksums, the oracle check, e2e, the peer-store probe,
# the other tree kinds, the N>1 chained iteration, placement and the reference arm
# under torchrun — not performance numbers.
O=gpurun_out/${1:-multi}; mkdir -p $O
export CCUBE_ALLOW_SHARED_GPU=1 CCUBE_BENCH_SHARED_GPU=1
R="timeout 900 python -m torch.distributed.run --nnodes=1 --master-addr 127.0.0.1"
IT="--iter-steps 2 --iter-rounds 1 --iter-warmup 1 --iter-batch 16 --extra-steps 3"
$R --nproc-per-node 2 --master-port 29511 bench.py --gpus 2 --steps 3 --warmup 3 --e2e-steps 2 \
  --max-elems 262144 --plan-placement $IT > $O/bench_n2.log 2>&1; echo "exit $?" >> $O/bench_n2.log
# >= 16 chunks of 256 KiB with AUTO channels on the double tree
$R --nproc-per-node 4 --master-port 29512 bench.py --gpus 4 --tree double --steps 3 --warmup 3 \
  --e2e-steps 2 --max-elems 1200000 --no-iter --extra-steps 3 > $O/bench_n4.log 2>&1; echo "exit $?" >> $O/bench_n4.log
$R --nproc-per-node 2 --master-port 29513 bench.py --impl reference --gpus 2 --steps 2 --warmup 1 \
  > $O/bench_ref_n2.log 2>&1; echo "exit $?" >> $O/bench_ref_n2.log

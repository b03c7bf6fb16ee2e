#!/bin/bash
# v19: data-warp readiness-spin back-off (CCUBE_BACKOFF_NS) at the bench workload, interleaved passes.
OUT=gpurun_out/bo; mkdir -p $OUT
for pass in 1 2 3; do
  for b in 64 0 16 32 128 256; do
    CCUBE_BACKOFF_NS=$b timeout 300 python bench.py --no-e2e --no-cpu-baseline --no-iter --no-clocks \
      | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'backoff_ns': $b, 'pass': $pass, 'ms': d['ms_per_step'], 'frac': d['roofline']['frac']}))" >> $OUT/sweep.jsonl
  done
done
CCUBE_BACKOFF_NS=0 timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "parity_small and float32" > $OUT/pytest_b0.log 2>&1; echo "exit $?" >> $OUT/pytest_b0.log

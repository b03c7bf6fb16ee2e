# UP lead window (back-pressure in loopback): sweep W, trace at the default, parity with a tight window
OUT=gpurun_out/s2b; mkdir -p $OUT
B="python bench.py --steps 100 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for rnd in 1 2; do
  for w in 0 12 16 24 32 48 64; do
    CCUBE_WINDOW=$w $B > $OUT/b_w${w}_$rnd.log 2>&1
    CCUBE_WINDOW=$w $B --tree double > $OUT/b_w${w}_double_$rnd.log 2>&1
  done
done
for w in 0 32; do
  CCUBE_WINDOW=$w CCUBE_TRACE_UP=1 python tools/pipeline_profile.py single > $OUT/pipeline_w$w.json 2> $OUT/pipe_w$w.err
done
CCUBE_WINDOW=1 timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "parity_small or channels or whole_buffer or special_values or repeated or gates" > $OUT/pytest_w1.log 2>&1; echo "exit $?" >> $OUT/pytest_w1.log
for w in 0 32; do
  CCUBE_WINDOW=$w python tools/size_sweep.py --ranks 8 --trees single --min-kib 512 --max-mib 64 --iters 20 > $OUT/sizes_w$w.jsonl 2> $OUT/sizes_w$w.err
done

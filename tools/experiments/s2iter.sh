# f3/f4 iteration sweep (3 nets x 4 batches x high/low bandwidth) at the session-2 build
OUT=gpurun_out/s2iter; mkdir -p $OUT
timeout 2700 python tools/iter_sweep.py > $OUT/iter_sweep.jsonl 2> $OUT/iter_sweep.err

OUT=gpurun_out/r2t; mkdir -p $OUT
B="python bench.py --steps 20 --warmup 5 --no-iter --no-cpu-baseline --no-extra --no-clocks --e2e-steps 10"
for n in 1 2 4; do $B --e2e-copy-streams $n > $OUT/b_cs$n.log 2>&1; done

# round-2 final evidence: full GPU suite, smoke, default bench line (driver command), ncu launch list + full capture
OUT=gpurun_out/r2s; mkdir -p $OUT
nvidia-smi > $OUT/nvidia-smi.txt 2>&1
timeout 2700 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.log 2>&1; echo "pytest exit $?" >> $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke exit $?" >> $OUT/smoke.log
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > $OUT/bench.log 2>&1; echo "bench exit $?" >> $OUT/bench.log
timeout 600 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > $OUT/bench_ref.log 2>&1; echo "ref exit $?" >> $OUT/bench_ref.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $OUT/launches.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-clocks --no-iter --no-extra > $OUT/launches_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tree_allreduce -s 3 -c 1 -o $OUT/prof python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-clocks --no-iter --no-extra > $OUT/prof_bench.log 2>&1
echo "ncu exit $?" >> $OUT/prof_bench.log

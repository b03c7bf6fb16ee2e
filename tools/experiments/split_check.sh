O=gpurun_out/split; mkdir -p $O
B="timeout 300 python bench.py --steps 100 --warmup 10 --no-e2e --no-cpu-baseline --no-iter --no-clocks"
for sp in 1 0; do for P in 8 4 2; do
  CCUBE_SPLIT_CONTROL=$sp $B --ranks $P > $O/bench_P${P}_s$sp.log 2>&1
done
CCUBE_SPLIT_CONTROL=$sp $B --tree double > $O/bench_P8d_s$sp.log 2>&1
CCUBE_SPLIT_CONTROL=$sp $B --tree rotated > $O/bench_P8r_s$sp.log 2>&1
done
python tools/pipeline_profile.py > $O/pipeline_s1.json 2> $O/pp.err
CCUBE_SPLIT_CONTROL=0 python tools/pipeline_profile.py > $O/pipeline_s0.json 2>> $O/pp.err
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "small or tma or channels or full_size_resnet" > $O/pytest.log 2>&1; echo "exit $?" >> $O/pytest.log

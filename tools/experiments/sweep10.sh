# v9: L2 eviction hints A/B, full GPU parity, iteration (chaining), ncu of the bench kernel
mkdir -p gpurun_out/sw10
for H in 0 1; do
CCUBE_L2_HINTS=$H timeout 300 python tools/sweep.py --ranks 8 --trees single,double --channels 0 --threads 256 --chunks 262144,1048576 > gpurun_out/sw10/P8_h$H.jsonl 2>&1
CCUBE_L2_HINTS=$H timeout 300 python tools/sweep.py --ranks 4 --trees single,double --channels 0 --threads 256 --chunks 262144 > gpurun_out/sw10/P4_h$H.jsonl 2>&1
CCUBE_L2_HINTS=$H timeout 300 python tools/sweep.py --ranks 2 --trees single,double --channels 0 --threads 256 --chunks 262144 > gpurun_out/sw10/P2_h$H.jsonl 2>&1
done
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/sw10/pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/sw10/pytest_gpu.log
timeout 600 python bench.py --mode iter --iter-channels 8 > gpurun_out/sw10/iter_c8.log 2>&1
timeout 600 python bench.py --mode iter --iter-channels 4 > gpurun_out/sw10/iter_c4.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tree_allreduce -s 3 -c 1 -o gpurun_out/sw10/prof python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-clocks --no-iter > gpurun_out/sw10/prof.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/sw10/launches.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-clocks --no-iter > gpurun_out/sw10/launches.log 2>&1

# multi-process IPC path on one GPU; iteration (chaining) with 4/8 channels; ncu of the bench kernel
mkdir -p gpurun_out/sw9
timeout 900 python -m pytest tests/test_gpu_multiproc.py -x -q > gpurun_out/sw9/pytest_mp.log 2>&1; echo "exit $?" >> gpurun_out/sw9/pytest_mp.log
timeout 600 python bench.py --mode iter --iter-channels 8 > gpurun_out/sw9/iter_c8.log 2>&1
timeout 600 python bench.py --mode iter --iter-channels 4 > gpurun_out/sw9/iter_c4.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tree_allreduce -s 3 -c 1 -o gpurun_out/sw9/prof python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-clocks --no-iter > gpurun_out/sw9/prof.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/sw9/launches.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-clocks --no-iter > gpurun_out/sw9/launches.log 2>&1

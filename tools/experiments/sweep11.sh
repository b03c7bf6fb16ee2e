# message-size sweep (configs[4]), turnaround (Fig 14b analogue), default bench line
mkdir -p gpurun_out/sw11
timeout 900 python tools/size_sweep.py --ranks 2,4,8 --trees single,double --overlap 1,0 > gpurun_out/sw11/sizes.jsonl 2> gpurun_out/sw11/sizes.err
timeout 300 python tools/turnaround.py > gpurun_out/sw11/turnaround.json 2> gpurun_out/sw11/turnaround.err
timeout 900 python bench.py > gpurun_out/sw11/bench.log 2>&1

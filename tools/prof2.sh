mkdir -p gpurun_out/prof2
CCUBE_DATAPATH=0 timeout 600 ncu --set full --clock-control none --import-source on -k regex:tree_allreduce -s 3 -c 1 -o gpurun_out/prof2/p2 python tools/sweep.py --ranks 2 --trees single --channels 0 --threads 256 --chunks 1048576 --tma 0 --iters 1 > gpurun_out/prof2/p2.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:stream_kernel -s 20 -c 1 -o gpurun_out/prof2/mb ./tools/bin/membench > gpurun_out/prof2/mb.log 2>&1

mkdir -p gpurun_out/sw1
python tools/sweep.py --trees single,double --channels 0 --threads 128,256 --chunks 65536,131072,262144,524288,1048576,2097152,4194304 > gpurun_out/sw1/chunks.jsonl 2>&1
python tools/sweep.py --trees single --channels 0,8,16,24,32 --threads 256 --chunks 262144,1048576 > gpurun_out/sw1/channels.jsonl 2>&1
python tools/sweep.py --trees single --channels 0 --threads 256 --chunks 262144,1048576 --transport push,pull --tma 0,1 > gpurun_out/sw1/transport.jsonl 2>&1
python tools/sweep.py --trees single --overlap 0,1 --channels 0 --threads 256 --chunks 262144 > gpurun_out/sw1/overlap.jsonl 2>&1

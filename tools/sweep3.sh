mkdir -p gpurun_out/sw3
for P in 2 3 4 8; do
python tools/sweep.py --ranks $P --trees single --channels 0,16,32,64 --threads 128,256 --chunks 1048576 > gpurun_out/sw3/P$P.jsonl 2>&1
done

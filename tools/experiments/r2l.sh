# final-code sweeps: sizes (LL + chunked), turnaround, N>1 plumbing on one GPU, NVLink counter tool plumbing
OUT=gpurun_out/r2l; mkdir -p $OUT
timeout 1500 python tools/size_sweep.py --ranks 2,4,8 --trees single,double,rotated --overlap 1,0 --min-kib 1 --max-mib 1024 > $OUT/sizes.jsonl 2> $OUT/sizes.err
timeout 300 python tools/turnaround.py > $OUT/turnaround.json 2> $OUT/turnaround.err
bash tools/experiments/multi_bench_check.sh r2l_multi
CCUBE_ALLOW_SHARED_GPU=1 CCUBE_BENCH_SHARED_GPU=1 timeout 400 bash tools/nvlink_counters.sh 2 --max-elems 262144 > $OUT/nvlink_shared.log 2>&1

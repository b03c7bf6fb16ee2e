# v11: fused SGD (f2), 7-data-warp variant A/B, VGG-16 + fused iterations
mkdir -p gpurun_out/sw13
timeout 2000 python -m pytest tests -m gpu -x -q > gpurun_out/sw13/pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/sw13/pytest_gpu.log
timeout 300 python tools/sweep.py --ranks 8 --trees single,double --channels 0 --threads 224,256 --chunks 262144 > gpurun_out/sw13/P8_threads.jsonl 2>&1
timeout 300 python tools/sweep.py --ranks 2 --trees single,double --channels 0 --threads 224,256 --chunks 262144 > gpurun_out/sw13/P2_threads.jsonl 2>&1
timeout 600 python bench.py --mode iter > gpurun_out/sw13/iter_r50.log 2>&1
timeout 600 python bench.py --mode iter --iter-fused-sgd > gpurun_out/sw13/iter_r50_fused.log 2>&1
timeout 900 python bench.py --mode iter --iter-model vgg16 --iter-rounds 2 > gpurun_out/sw13/iter_vgg.log 2>&1

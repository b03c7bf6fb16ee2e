set -x
OUT=gpurun_out/r2a; mkdir -p $OUT
nvidia-smi > $OUT/nvidia-smi.txt 2>&1
python -c "import torch;print(torch.cuda.get_device_properties(0))" > $OUT/dev.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_multiproc.py -x -q > $OUT/pytest_multiproc.log 2>&1; echo "exit $?" >> $OUT/pytest_multiproc.log
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "gates_each_layer or parity_small or channels" > $OUT/pytest_parity_subset.log 2>&1; echo "exit $?" >> $OUT/pytest_parity_subset.log
timeout 300 python tools/pipeline_profile.py single > $OUT/pipeline_single.json 2> $OUT/pipeline.err
timeout 300 python bench.py --steps 50 --warmup 5 --no-iter --no-cpu-baseline > $OUT/bench.log 2>&1

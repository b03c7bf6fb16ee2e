# round 2: streaming ceilings (membench2/3, torch copy), tree kernel without its
# dependencies (CCUBE_DEBUG_NODEP, timing only), special-value + whole-buffer parity
OUT=gpurun_out/r2c; mkdir -p $OUT
./tools/bin/membench3 256 > $OUT/membench3_256.jsonl 2>&1
./tools/bin/membench3 1024 > $OUT/membench3_1024.jsonl 2>&1
./tools/bin/membench2 > $OUT/membench2.jsonl 2>&1
python - > $OUT/torch_copy.jsonl 2>&1 <<'PY'
import torch, json
for mb in (256, 1024, 2048):
    a = torch.empty(mb << 20, dtype=torch.uint8, device="cuda"); b = torch.empty_like(a)
    best = 1e9
    for i in range(8):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); b.copy_(a); e1.record(); torch.cuda.synchronize()
        if i: best = min(best, e0.elapsed_time(e1))
    print(json.dumps({"variant": "torch_copy", "bytes_per_buffer": mb << 20, "ms": best,
                      "gbs": 2 * (mb << 20) / best / 1e6}))
PY
B="python bench.py --steps 50 --warmup 5 --no-iter --no-e2e --no-cpu-baseline --no-extra --no-clocks"
for tree in single double; do
  $B --tree $tree > $OUT/bench_$tree.log 2>&1
  CCUBE_DEBUG_NODEP=1 $B --tree $tree > $OUT/bench_${tree}_nodep.log 2>&1
done
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "special or whole_buffer or keeps_subnormals" > $OUT/pytest_special.log 2>&1; echo "exit $?" >> $OUT/pytest_special.log

"""Chained-iteration sweeps (SURVEY §8 f3 + f4; Fig 13 / Fig 15 analogues,
P:L272): models x per-GPU batch x link bandwidth, modes compute / B /
C1 / C2 / CC of bench.py's run_iteration, one JSON line per configuration.

  --models resnet50,vgg16,zfnet   the paper's three networks (ZFNet-like, workloads.py)
  --batches 16,32,64,128          "We also varied the batch size"
  --bandwidth high,low            the paper's low-bandwidth setting "reducing the
                                  number of threads allocated to the AllReduce
                                  kernel": high = the iteration's full
                                  channel count, low = a quarter of its CTAs.

In loopback (one GPU, P logical ranks) the full setting is a fixed channel count
(16 channels, 16 x 7 + 4 = 116 CTAs at P = 8): the automatic count would give the
AllReduce every SM and leave the forward nothing to overlap on.  The low setting
is a quarter of that many channels, hence a quarter of the AllReduce CTAs.

    python tools/iter_sweep.py > profiles/r02/iter_sweep.jsonl
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--models", default="resnet50,vgg16,zfnet")
    p.add_argument("--batches", default="16,32,64,128")
    p.add_argument("--bandwidth", default="high,low")
    p.add_argument("--high-channels", type=int, default=16)
    p.add_argument("--ranks", type=int, default=8)
    p.add_argument("--steps", type=int, default=10)
    p.add_argument("--rounds", type=int, default=3)
    a = p.parse_args()
    import torch
    torch.cuda.set_device(0)
    for model in a.models.split(","):
        for batch in [int(x) for x in a.batches.split(",")]:
            for bwm in a.bandwidth.split(","):
                ch = a.high_channels if bwm == "high" else max(1, a.high_channels // 4)
                args = bench.parse_args_list([
                    "--iter-model", model, "--iter-batch", str(batch), "--iter-channels", str(ch),
                    "--iter-steps", str(a.steps), "--iter-rounds", str(a.rounds),
                    "--ranks", str(a.ranks)])
                try:
                    it = bench.run_iteration(args, a.ranks)
                except Exception as e:  # noqa: BLE001
                    it = {"error": repr(e)}
                print(json.dumps({"model": model, "batch_per_gpu": batch, "bandwidth": bwm,
                                  "channels": ch, "P": a.ranks, "iteration": it}), flush=True)
                torch.cuda.empty_cache()


if __name__ == "__main__":
    main()

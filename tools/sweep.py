"""Parameter sweep of the loopback AllReduce (device time, CUDA events).

    python tools/sweep.py --workload resnet50 --channels 8,16 --threads 256,512 --chunks 262144
"""
import argparse
import itertools
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_sanghoonsk23_b200 import ccube, workloads  # noqa: E402


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--workload", default="resnet50")
    p.add_argument("--dtype", default="float32")
    p.add_argument("--ranks", type=int, default=8)
    p.add_argument("--trees", default="single")
    p.add_argument("--overlap", default="1")
    p.add_argument("--channels", default="8")
    p.add_argument("--threads", default="512")
    p.add_argument("--chunks", default=str(256 << 10))
    p.add_argument("--iters", type=int, default=20)
    p.add_argument("--transport", default="auto")
    p.add_argument("--bytes", type=int, default=0, help="override buffer bytes per rank")
    a = p.parse_args()
    tdt = {"float32": torch.float32, "bfloat16": torch.bfloat16, "int32": torch.int32}[a.dtype]
    es = torch.tensor([], dtype=tdt).element_size()
    count = a.bytes // es if a.bytes else workloads.total_elems(a.workload)
    P = a.ranks
    bufs = [torch.randn(count, device="cuda").to(tdt) for _ in range(P)]
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    s = torch.cuda.Stream()
    for tree, ov, ch, th, cb, tp in itertools.product(
            a.trees.split(","), a.overlap.split(","), a.channels.split(","), a.threads.split(","),
            a.chunks.split(","), a.transport.split(",")):
        try:
            ccube.init_loopback(P, tree, int(cb))
            ccube.set_channels(int(ch))
            ccube.set_threads(int(th))
            ccube.set_overlap(bool(int(ov)))
            ccube.set_transport(tp)
            ms = []
            for i in range(a.iters + 3):
                with torch.cuda.stream(s):
                    flush.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                ccube.allreduce_tree_local(bufs, stream=s)
                e1.record(s)
                torch.cuda.synchronize()
                if i >= 3:
                    ms.append(e0.elapsed_time(e1))
            med = float(np.median(ms))
            nbytes = count * es
            busbw = nbytes / (med / 1e3) / 1e9 * 2 * (P - 1) / P
            hbm = 2 * P * nbytes / (med / 1e3) / 1e9
            print(json.dumps({"P": P, "tree": tree, "transport": tp, "overlap": int(ov),
                              "channels": ccube.get_info()["last_channels"],
                              "ctas": ccube.get_info()["last_ctas"],
                              "threads": int(th), "chunk": int(cb), "ms": round(med, 4),
                              "busbw": round(busbw, 1), "hbm_algo_gbs": round(hbm, 1)}),
                  flush=True)
        except ccube.CCubeError as e:
            print(json.dumps({"tree": tree, "channels": ch, "threads": th, "chunk": cb,
                              "error": str(e)}), flush=True)
        finally:
            try:
                ccube.finalize()
            except ccube.CCubeError:
                pass


if __name__ == "__main__":
    main()

"""Message-size sweep (BASELINE.json configs[4]): loopback tree AllReduce busbw vs
bytes per rank, 1 KiB .. 1 GiB, at P = 2/4/8 logical ranks on one B200, single vs
double tree, C1 vs B.  Device time per call: CUDA events on the launching stream
around one launch (> 1 MiB) or around --inner back-to-back launches (<= 1 MiB, as
nccl-tests does, since an event pair resolves only ~2 us), median of --iters after
--warmup.  nccl-tests convention:
buffers are NOT flushed between calls (sizes below L2 run from L2), and busbw =
algbw * 2(P-1)/P.

    python tools/size_sweep.py --ranks 2,4,8 --trees single,double --overlap 1,0 \
        --min-kib 1 --max-mib 1024 > sizes.jsonl
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_sanghoonsk23_b200 import ccube  # noqa: E402


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--ranks", default="2,4,8")
    p.add_argument("--trees", default="single,double")
    p.add_argument("--overlap", default="1,0")
    p.add_argument("--chunk-bytes", type=int, default=256 << 10)
    p.add_argument("--min-kib", type=int, default=1)
    p.add_argument("--max-mib", type=int, default=1024)
    p.add_argument("--iters", type=int, default=20)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--inner", type=int, default=20,
                   help="calls per timed pair for messages <= 1 MiB")
    p.add_argument("--protocol", default="ll,chunked",
                   help="ll: one-chunk calls on the LL kernel (default); chunked: LL off")
    a = p.parse_args()
    sizes = []
    b = a.min_kib << 10
    while b <= a.max_mib << 20:
        sizes.append(b)
        b *= 2
    s = torch.cuda.Stream()
    for P in [int(x) for x in a.ranks.split(",")]:
        bufs = [torch.randn(sizes[-1] // 4, device="cuda") for _ in range(P)]
        for tree in a.trees.split(","):
            ccube.init_loopback(P, tree, a.chunk_bytes)
            try:
                for ov, proto in [(int(o), pr) for o in a.overlap.split(",")
                                  for pr in a.protocol.split(",")]:
                    ccube.set_overlap(bool(ov))
                    ccube.set_protocol(proto == "ll")
                    for nbytes in sizes:
                        if proto == "chunked" and nbytes > a.chunk_bytes and "ll" in a.protocol:
                            continue   # same kernel as the LL run's point
                        count = nbytes // 4
                        # small messages: `inner` back-to-back calls between two events
                        # (an event pair alone resolves ~2 us); device time per call
                        inner = a.inner if nbytes <= (1 << 20) else 1
                        evs = [(torch.cuda.Event(enable_timing=True),
                                torch.cuda.Event(enable_timing=True))
                               for _ in range(a.iters + a.warmup)]
                        for e0, e1 in evs:
                            e0.record(s)
                            for _ in range(inner):
                                ccube.allreduce_tree_local(bufs, count=count, stream=s)
                            e1.record(s)
                        torch.cuda.synchronize()
                        ms = [e0.elapsed_time(e1) / inner for e0, e1 in evs[a.warmup:]]
                        med = float(np.median(ms))
                        alg = nbytes / (med / 1e3) / 1e9
                        info = ccube.get_info()
                        print(json.dumps({
                            "P": P, "tree": tree, "mode": "C1" if ov else "B", "bytes": nbytes,
                            "protocol": "ll" if info["last_ll"] else "chunked",
                            "chunk_bytes": a.chunk_bytes, "channels": info["last_channels"],
                            "calls_per_timing": inner,
                            "ctas": info["last_ctas"], "us": round(med * 1e3, 2),
                            "us_p10_p90": [round(float(np.percentile(ms, q)) * 1e3, 2)
                                           for q in (10, 90)],
                            "algbw": round(alg, 2), "busbw": round(alg * 2 * (P - 1) / P, 2),
                            "hbm_algo_gbs": round(2 * P * nbytes / (med / 1e3) / 1e9, 1)}),
                            flush=True)
            finally:
                ccube.finalize()
        del bufs
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()

"""Where the P = 8 loopback pipeline spends its time: landing trace of the bench
workload (ResNet-50 gradient set, single tree, C1, auto channels).  For every rank,
the time chunk k landed there (max over channel slices), relative to the first
landing anywhere, plus the steady-state interval per chunk.  The root's landings
are its reduce-up completions; the lag of each level behind its parent shows which
stage sets the pace.

    python tools/pipeline_profile.py > pipeline.json
"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_sanghoonsk23_b200 import ccube, workloads  # noqa: E402


def main(P=8, tree="single", chunk=256 << 10, reps=5):
    count = workloads.total_elems("resnet50")
    bufs = [torch.randn(count, device="cuda") for _ in range(P)]
    pristine = [b.clone() for b in bufs]
    ccube.init_loopback(P, tree, chunk)
    out = {"P": P, "tree": tree, "count": count, "chunk_bytes": chunk}
    try:
        ccube.allreduce_tree_local(bufs)
        torch.cuda.synchronize()
        J = ccube.get_info()["last_channels"]
        T = 1 if tree == "single" else 2
        K = -(-count * 4 // chunk)
        kmax = -(-K // T)
        trace = torch.zeros(P * T * kmax * J, dtype=torch.int64, device="cuda")
        ccube.set_trace(trace, kmax)
        lands = []
        for _ in range(reps):
            for b, p in zip(bufs, pristine):
                b.copy_(p)
            trace.zero_()
            torch.cuda.synchronize()
            ccube.allreduce_tree_local(bufs)
            torch.cuda.synchronize()
            tr = trace.view(P, T, kmax, J).cpu().numpy().astype(np.int64)
            t0 = tr[tr > 0].min()
            lands.append((tr.max(axis=3) - t0) / 1e3)   # us, [P, T, kmax]
        ccube.set_trace(None, 0)
        land = np.median(np.stack(lands), axis=0)
        ks = [0, 1, 5, 10, 50, 100, 200, 300, kmax - 1]
        out["channels"] = J
        out["landing_us"] = {f"rank{r}": {str(k): round(float(land[r, 0, k]), 2) for k in ks}
                             for r in range(P)}
        lo, hi = kmax // 4, kmax - 1
        out["steady_us_per_chunk"] = {
            f"rank{r}": round(float((land[r, 0, hi] - land[r, 0, lo]) / (hi - lo)), 4)
            for r in range(P)}
        # per-slice spread: how far apart the channels of one chunk land (rank 1)
        tr_last = (np.stack(lands)[-1])
        out["last_landing_us"] = round(float(land.max()), 2)
    finally:
        ccube.finalize()
    print(json.dumps(out))


if __name__ == "__main__":
    main(tree=sys.argv[1] if len(sys.argv) > 1 else "single")

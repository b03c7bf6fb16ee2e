"""Where the P = 8 loopback pipeline spends its time: landing trace of the bench
workload (ResNet-50 gradient set, single tree, C1, auto channels).

For every rank: the time chunk k landed there (max over channel slices), and with
CCUBE_TRACE_UP=1 also the time its reduce-up partial of chunk k was handed to the
parent; all relative to the first traced event of the launch.  Also the
steady-state interval per chunk of each stage and the launch's duration (CUDA
events around it, which also include the launch latency).

    CCUBE_TRACE_UP=1 python tools/pipeline_profile.py [single|double] > pipeline.json
"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_sanghoonsk23_b200 import ccube, workloads  # noqa: E402


def main(P=8, tree="single", chunk=256 << 10, reps=5):
    up = os.environ.get("CCUBE_TRACE_UP") == "1"
    count = workloads.total_elems("resnet50")
    bufs = [torch.randn(count, device="cuda") for _ in range(P)]
    pristine = [b.clone() for b in bufs]
    ccube.init_loopback(P, tree, chunk)
    out = {"P": P, "tree": tree, "count": count, "chunk_bytes": chunk, "trace_up": up}
    try:
        ccube.allreduce_tree_local(bufs)
        torch.cuda.synchronize()
        J = ccube.get_info()["last_channels"]
        T = {"single": 1, "double": 2}[tree]
        K = -(-count * 4 // chunk)
        kmax = -(-K // T)
        n = P * T * kmax * J
        trace = torch.zeros(n * (2 if up else 1), dtype=torch.int64, device="cuda")
        ccube.set_trace(trace, kmax)
        lands, ups, kern = [], [], []
        for _ in range(reps):
            for b, p in zip(bufs, pristine):
                b.copy_(p)
            trace.zero_()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            ccube.allreduce_tree_local(bufs, stream=torch.cuda.current_stream())
            e1.record()
            torch.cuda.synchronize()
            kern.append(e0.elapsed_time(e1) * 1e3)
            tr = trace.cpu().numpy().astype(np.int64)
            t0 = tr[tr > 0].min()
            land = tr[:n].reshape(P, T, kmax, J)
            lands.append((land.max(axis=3) - t0) / 1e3)   # us, [P, T, kmax]
            if up:
                u = tr[n:].reshape(P, T, kmax, J)
                um = np.where(u.max(axis=3) > 0, (u.max(axis=3) - t0) / 1e3, np.nan)
                ups.append(um)
        ccube.set_trace(None, 0)
        land = np.median(np.stack(lands), axis=0)
        ks = sorted({k for k in (0, 1, 5, 10, 50, 100, 200, 300) if k < kmax} | {kmax - 1})
        out["channels"] = J
        out["kernel_us_events"] = float(np.median(kern))
        out["landing_us"] = {f"rank{r}": {str(k): round(float(land[r, 0, k]), 2) for k in ks}
                             for r in range(P)}
        lo, hi = kmax // 4, kmax - 1
        out["steady_us_per_chunk"] = {
            f"rank{r}": round(float((land[r, 0, hi] - land[r, 0, lo]) / (hi - lo)), 4)
            for r in range(P)}
        out["last_landing_us"] = round(float(land.max()), 2)
        if up:
            u = np.nanmedian(np.stack(ups), axis=0)
            out["up_handoff_us"] = {
                f"rank{r}": {str(k): round(float(u[r, 0, k]), 2) for k in ks}
                for r in range(P) if not np.isnan(u[r, 0, 0])}
            out["up_steady_us_per_chunk"] = {
                f"rank{r}": round(float((u[r, 0, hi] - u[r, 0, lo]) / (hi - lo)), 4)
                for r in range(P) if not np.isnan(u[r, 0, 0])}
    finally:
        ccube.finalize()
    print(json.dumps(out))


if __name__ == "__main__":
    main(tree=sys.argv[1] if len(sys.argv) > 1 else "single")

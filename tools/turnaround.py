"""Gradient turnaround, B vs C1 (the Fig 14(b) analogue): time from the
first landing anywhere to the moment chunk 0 has landed on EVERY rank, for a
64 MiB fp32 buffer cut into 256 chunks of 256 KiB, P = 8 loopback ranks.  Uses
the library's landing trace (%globaltimer at every Enqueue-Semaphore publish).

    python tools/turnaround.py > turnaround.json
"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_sanghoonsk23_b200 import ccube  # noqa: E402


def main(P=8, nbytes=64 << 20, chunk=256 << 10, reps=10):
    K = nbytes // chunk
    out = {"P": P, "bytes": nbytes, "chunk_bytes": chunk, "chunks": K, "reps": reps}
    bufs = [torch.randn(nbytes // 4, device="cuda") for _ in range(P)]
    for tree in ("single", "double"):
        ccube.init_loopback(P, tree, chunk)
        try:
            T = 2 if tree == "double" else 1
            kmax = (K + T - 1) // T
            for ov in (0, 1):
                ccube.set_overlap(bool(ov))
                ccube.allreduce_tree_local(bufs)   # warm-up, picks the channel count
                torch.cuda.synchronize()
                J = ccube.get_info()["last_channels"]
                trace = torch.zeros(P * T * kmax * J, dtype=torch.int64, device="cuda")
                ccube.set_trace(trace, kmax)
                turn, total = [], []
                for _ in range(reps):
                    trace.zero_()
                    ccube.allreduce_tree_local(bufs)
                    torch.cuda.synchronize()
                    tr = trace.view(P, T, kmax, J).cpu().numpy().astype(np.int64)
                    land = tr.max(axis=3)          # a chunk landed when all its slices did
                    t0 = tr[tr > 0].min()
                    # global chunk 0 is tree 0's local chunk 0
                    turn.append((land[:, 0, 0].max() - t0) / 1e3)
                    total.append((land.max() - t0) / 1e3)
                ccube.set_trace(None, 0)
                out[f"{tree}_{'C1' if ov else 'B'}"] = {
                    "turnaround_us": float(np.median(turn)), "last_landing_us": float(np.median(total)),
                    "channels": J}
        finally:
            ccube.finalize()
    for tree in ("single", "double"):
        b, c = out[f"{tree}_B"]["turnaround_us"], out[f"{tree}_C1"]["turnaround_us"]
        out[f"{tree}_turnaround_ratio_B_over_C1"] = b / c if c > 0 else None
    print(json.dumps(out))


if __name__ == "__main__":
    main()

"""Fig 16's three computation/communication patterns on
the gradient queue: how much exposed communication chaining removes when

  Case 1: forward compute per layer DECREASES and gradient size INCREASES with the
          layer index (CNNs, Fig 17) — the gates of early layers open early;
  Case 2: compute INCREASES with the layer index — "bubbles": layer l's forward is
          done before layer l+1's gradients land;
  Case 3: gradient size is front-loaded (large early layers) — the first gates open
          late, the gradient turnaround is pushed back.

A synthetic data-parallel iteration, loopback (P logical ranks on one GPU, 4
AllReduce channels as in bench.py's iteration): L layers; layer l owns S_l fp32
gradients (the gradient queue) and its forward is n_l bf16 GEMMs of 512x4096x4096 (a
stand-in for the layer's compute; cuBLAS, not the hot path); the backward is a
fixed GEMM block (2x the forward) followed by writing every rank's gradients.
The forward is run at 64, 16 and 8 GEMMs in total (compute >>, ~=, < the
AllReduce).  Modes: compute only, C1 unchained (the forward waits for the whole AllReduce), CC
(C1 + one ccube_gradq_wait per layer before its forward).  Totals (bytes,
FLOPs) are the same in every case; only their distribution over the layers moves.

    python tools/case_study.py > case_study.json
"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_sanghoonsk23_b200 import ccube  # noqa: E402

L = 16
TOTAL_ELEMS = 25_557_032           # ResNet-50's gradient count (102 MB fp32)
TOTAL_GEMMS = 64                   # forward GEMMs per iteration
N = 4096


def profile(case, total_gemms=TOTAL_GEMMS):
    up = np.array([2.0 ** (l / 3) for l in range(L)])     # increasing with the layer index
    size = up if case in (1, 2) else up[::-1]
    comp = up[::-1] if case in (1, 3) else up
    s = np.maximum(1, np.round(size / size.sum() * TOTAL_ELEMS)).astype(np.int64)
    s[-1] += TOTAL_ELEMS - s.sum()
    # compute in units of 512-row GEMMs (1/8 of a 4096^3 GEMM), at least one per layer
    n = np.maximum(1, np.round(comp / comp.sum() * total_gemms * 8)).astype(np.int64)
    return [int(x) for x in s], [int(x) for x in n]


def run_case(case, total_gemms=TOTAL_GEMMS, P=8, rank=1, channels=4, steps=10, warmup=2,
             rounds=3, chunk=256 << 10):
    dev = torch.device("cuda", 0)
    sizes, gemms = profile(case, total_gemms)
    ends = list(np.cumsum(sizes))
    count = ends[-1]
    bufs = [torch.zeros(count, device=dev) for _ in range(P)]
    grad_src = torch.randn(count, device=dev)
    a = torch.randn(N, N, device=dev, dtype=torch.bfloat16)
    b = torch.randn(N, N, device=dev, dtype=torch.bfloat16)
    c = torch.empty(N, N, device=dev, dtype=torch.bfloat16)
    comp, comm = torch.cuda.Stream(), torch.cuda.Stream()
    ccube.init_loopback(P, "single", chunk)
    ccube.set_channels(channels)
    ccube.gradq_set_layers(ends)
    modes = ("compute", "C1", "CC")
    runs = {m: [] for m in modes}

    def one(mode):
        with torch.cuda.stream(comp):
            for l in range(L):                      # forward of the next iteration
                if mode == "CC":
                    ccube.gradq_wait_local(rank, l, stream=comp)
                q, r = divmod(gemms[l], 8)
                for _ in range(q):
                    torch.mm(a, b, out=c)
                if r:
                    torch.mm(a[: 512 * r], b, out=c[: 512 * r])
            comp.wait_stream(comm)                  # the AllReduce is done with the queue
            for _ in range(2 * sum(gemms) // 8):    # backward
                torch.mm(a, b, out=c)
            for x in bufs:                          # every rank's gradients
                x.copy_(grad_src)
        if mode != "compute":
            comm.wait_stream(comp)
            ccube.allreduce_tree_local(bufs, stream=comm)
            if mode == "C1":
                comp.wait_stream(comm)

    try:
        ccube.set_overlap(True)
        for _ in range(rounds):
            for mode in modes:
                for _ in range(warmup):
                    one(mode)
                torch.cuda.synchronize()
                e0 = torch.cuda.Event(enable_timing=True)
                e1 = torch.cuda.Event(enable_timing=True)
                e0.record(comp)
                for _ in range(steps):
                    one(mode)
                comp.wait_stream(comm)
                e1.record(comp)
                torch.cuda.synchronize()
                runs[mode].append(e0.elapsed_time(e1) / steps)
    finally:
        ccube.finalize()
    ms = {m: float(np.median(v)) for m, v in runs.items()}
    exp = {m: ms[m] - ms["compute"] for m in ("C1", "CC")}
    return {"case": case, "total_gemms": total_gemms, "layer_elems": sizes,
            "layer_gemm_units_512_rows": gemms, "ms": ms,
            "exposed_ms": exp, "runs_ms": runs,
            "exposed_cut_CC_vs_C1": (1 - exp["CC"] / exp["C1"]) if exp["C1"] > 0 else None}


def main():
    torch.cuda.set_device(0)
    out = {"P": 8, "tree": "single", "channels": 4, "gemm": f"bf16 {N}^3",
           "note": "loopback; synthetic layers; Fig 16 Case 1/2/3 (P:L326-330)",
           "cases": [run_case(c, g) for g in (TOTAL_GEMMS, 16, 8) for c in (1, 2, 3)]}
    print(json.dumps(out))


if __name__ == "__main__":
    main()

"""α–β model fit of the measured tree AllReduce (the Fig 12(b)
analogue: "the measured ... closely matches" the model).

The paper's step model (eq 3; overlapped form eq 6): a tree
of depth D moving K chunks of C bytes takes
    B  (non-overlapped):  2(K + D - 1) steps       (reading R6)
    C1 (overlapped):       K + 2D - 1  steps
each step costing alpha + beta * C.  With T trees each tree carries K_t = ceil(K/T)
chunks and the trees run concurrently.  One term is added to the paper's model:
a fixed per-call cost t0 (kernel launch and teardown, which the paper's
persistent-kernel setting does not pay per step).  This tool fits (t0, alpha,
beta) per (P, tree) to the C1 points of a size sweep by least squares on the
relative error, then PREDICTS the B points with the same three numbers and
reports predicted vs measured B/C1.

    python tools/model_fit.py profiles/r01/sizes_v9.jsonl > profiles/r01/model_fit.json
"""
import json
import math
import sys
from collections import defaultdict

import numpy as np

DEPTH = {1: 0, 2: 1, 3: 2, 4: 2, 5: 3, 6: 3, 7: 3, 8: 3}   # btree depth in edges (R1)
NTREES = {"single": lambda P: 1, "double": lambda P: 2, "rotated": lambda P: P}


def steps(mode, K, D):
    return 2 * (K + D - 1) if mode == "B" else K + 2 * D - 1


def main(path):
    rows = [json.loads(l) for l in open(path) if l.startswith("{")]
    groups = defaultdict(list)
    for r in rows:
        groups[(r["P"], r["tree"])].append(r)
    out = {"source": path, "fits": []}
    for (P, tree), rs in sorted(groups.items()):
        T = NTREES[tree](P)
        D = DEPTH[P]

        def design(r):
            C = min(r["chunk_bytes"], r["bytes"])
            K = math.ceil(r["bytes"] / r["chunk_bytes"])
            Kt = math.ceil(K / T)
            n = steps(r["mode"], Kt, D)
            return 1.0, n, n * C

        c1 = [r for r in rs if r["mode"] == "C1"]
        if len(c1) < 3:
            continue
        A = np.array([design(r) for r in c1], dtype=float)
        y = np.array([r["us"] for r in c1], dtype=float)
        w = 1.0 / y                                   # relative-error weighting
        (t0, alpha, beta), *_ = np.linalg.lstsq(A * w[:, None], y * w, rcond=None)
        coef = np.array([t0, alpha, beta])
        pred = A @ coef
        r2 = 1 - float(np.sum((y - pred) ** 2) / np.sum((y - y.mean()) ** 2))
        by_size = {r["bytes"]: r for r in rs if r["mode"] == "B"}
        cmp = []
        for r in c1:
            b = by_size.get(r["bytes"])
            if not b:
                continue
            pb = np.array(design(b)) @ coef
            pc = np.array(design(r)) @ coef
            cmp.append({"bytes": r["bytes"], "measured_B_over_C1": b["us"] / r["us"],
                        "model_B_over_C1": float(pb / pc), "model_B_us": float(pb),
                        "measured_B_us": b["us"]})
        out["fits"].append({
            "P": P, "tree": tree, "trees": T, "depth": D, "t0_us": float(t0),
            "alpha_us": float(alpha),
            "beta_us_per_byte": float(beta),
            "step_bw_gbs": (1e-3 / float(beta)) if beta > 0 else None,
            "r2_c1": r2, "max_rel_err_c1": float(np.max(np.abs(pred - y) / y)),
            "points": len(c1), "b_vs_c1": cmp})
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main(sys.argv[1])

"""Placement planning (reading R19; oracle — test infrastructure only).

Paper basis: on the DGX-1 hybrid cube-mesh some GPU pairs have no direct NVLink
and C-Cube routes those tree edges through detour GPUs (§IV).  On an
NVSwitch box every pair has a direct path, so the only topology decision left is
which physical rank hosts which tree position ("root placement" in the north
star), made against the measured peer bandwidth.

Cost model (R19): every tree t of the kind carries 1/T of the buffer; each tree
edge (child c, parent p) carries that share up (c -> p) and down (p -> c).  With
bw[i][j] the measured i -> j bandwidth, a placement's cost is
    max over directed pairs (i, j) with load > 0 of load(i, j) / bw[i][j]
(the slowest edge sets the pipeline's rate, eq 3's beta term per edge).  The plan
is the permutation of least cost; ties go to the lexicographically smallest
permutation, so uniform bandwidth gives the identity.  Brute force over P!.
"""

from fractions import Fraction
from itertools import permutations
from typing import List, Sequence

from .trees import trees


def edge_loads(P: int, kind: str, perm: Sequence[int]) -> List[List[Fraction]]:
    """load[i][j] = fraction of the buffer sent from rank i to rank j."""
    ts = trees(P, kind, perm)
    share = Fraction(1, len(ts))
    load = [[Fraction(0)] * P for _ in range(P)]
    for t in ts:
        for c in range(P):
            p = t.parent[c]
            if p >= 0:
                load[c][p] += share
                load[p][c] += share
    return load


def cost(P: int, kind: str, bw: Sequence[Sequence[float]], perm: Sequence[int]) -> float:
    load = edge_loads(P, kind, perm)
    worst = 0.0
    for i in range(P):
        for j in range(P):
            if load[i][j] > 0:
                if bw[i][j] <= 0:
                    return float("inf")
                worst = max(worst, float(load[i][j]) / bw[i][j])
    return worst


def plan(P: int, kind: str, bw: Sequence[Sequence[float]]) -> List[int]:
    """Least-cost placement.  A placement relabels the identity trees, so its loads
    are load_perm[perm[i]][perm[j]] = load_id[i][j] (checked against edge_loads by
    the tests); that keeps the P! search cheap."""
    base = edge_loads(P, kind, list(range(P)))
    edges = [(i, j, float(base[i][j])) for i in range(P) for j in range(P) if base[i][j] > 0]
    best, best_cost = list(range(P)), None
    for perm in permutations(range(P)):      # lexicographic order, identity first
        c = 0.0
        for i, j, ld in edges:
            b = bw[perm[i]][perm[j]]
            c = max(c, float("inf") if b <= 0 else ld / b)
        if best_cost is None or c < best_cost:
            best, best_cost = list(perm), c
    return best

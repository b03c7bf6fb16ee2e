"""Linear alpha-beta cost models and NVSwitch port loads (oracle; test infrastructure only).

Paper basis (§II-C, §III-C): N message size, K chunks, P processors, alpha latency,
beta = 1/bandwidth.

  eq 1  T_AllGather = (P-1)(alpha + beta N/P)
  eq 2  T_ring      = 2(P-1) alpha + 2((P-1)/P) beta N
  eq 3  T_reduction = T_broadcast = (log P + K)(alpha + beta N/K)
  eq 4  K_opt       = sqrt(log P beta N / alpha)
  eq 6  T_tree      = 2 log P alpha + 2 beta N + 4 sqrt(alpha beta N log P)
  eq 7  T_C1        = 2 log P alpha + beta N + 3 sqrt(alpha beta N log P)
  steps: 2(log P + K) baseline vs 2 log P + K overlapped

Reading R7: eq 7's coefficient 3 does not follow from substituting the optimum of
(2 log P + K)(alpha + beta N / K), which gives 2*sqrt(2) ~= 2.83; ``t_c1_exact``
is that derivation and eq 7 is kept verbatim as ``t_c1_eq7``.  log is base 2
(tree depth).

Port loads (NVSwitch reading of §IV): with one port per GPU, the
bytes rank v sends per direction in one AllReduce are
sum_t (#children_t(v) + [v != root_t]) * N_t.
"""

import math
from typing import List

from .trees import trees as build_trees


def t_allgather(P: int, N: float, alpha: float, beta: float) -> float:
    return (P - 1) * (alpha + beta * N / P)


def t_ring(P: int, N: float, alpha: float, beta: float) -> float:
    return 2 * (P - 1) * alpha + 2 * ((P - 1) / P) * beta * N


def t_phase(P: int, N: float, K: float, alpha: float, beta: float) -> float:
    """eq 3: one phase (reduction or broadcast) of the pipelined tree."""
    return (math.log2(P) + K) * (alpha + beta * N / K)


def k_opt(P: int, N: float, alpha: float, beta: float) -> float:
    return math.sqrt(math.log2(P) * beta * N / alpha)


def t_tree(P: int, N: float, alpha: float, beta: float) -> float:
    """eq 6 (baseline B at K_opt)."""
    L = math.log2(P)
    return 2 * L * alpha + 2 * beta * N + 4 * math.sqrt(alpha * beta * N * L)


def t_c1_eq7(P: int, N: float, alpha: float, beta: float) -> float:
    """eq 7 verbatim."""
    L = math.log2(P)
    return 2 * L * alpha + beta * N + 3 * math.sqrt(alpha * beta * N * L)


def t_c1_steps(P: int, N: float, K: float, alpha: float, beta: float) -> float:
    """Overlapped tree with 2 log P + K steps of (alpha + beta N/K)."""
    return (2 * math.log2(P) + K) * (alpha + beta * N / K)


def t_c1_exact(P: int, N: float, alpha: float, beta: float) -> float:
    """min over K of t_c1_steps: 2 log P alpha + beta N + 2 sqrt(2 alpha beta N log P)."""
    L = math.log2(P)
    return 2 * L * alpha + beta * N + 2 * math.sqrt(2 * alpha * beta * N * L)


def port_loads(P: int, kind: str, N: float) -> List[float]:
    """Bytes each rank sends per direction for one AllReduce of N bytes."""
    ts = build_trees(P, kind)
    share = N / len(ts)
    out = [0.0] * P
    for tr in ts:
        for v in range(P):
            out[v] += (len(tr.children[v]) + (1 if v != tr.root else 0)) * share
    return out


def busbw_ceiling(P: int, kind: str, port_gbs: float) -> float:
    """busbw = algbw * 2(P-1)/P bounded by the busiest port (overlapped modes)."""
    if P < 2:
        return float("inf")
    worst = max(port_loads(P, kind, 1.0))
    return port_gbs / worst * 2 * (P - 1) / P

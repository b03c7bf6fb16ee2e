"""Placement from measured peer bandwidth (reading R19; §IV).

On the paper's DGX-1 hybrid cube-mesh, missing GPU pairs forced detour routes.
On an NVSwitch box every pair has a direct path, so the remaining decision is
which rank hosts which tree position; ``plan(pg)`` measures the P x P peer
bandwidth matrix over the process group and asks the library's planner
(``ccube_plan_placement``) for the least-cost permutation, which every rank then
passes to ``ccube.set_placement`` before ``ccube.init_distributed``.  Init-time
only: nothing here runs on the AllReduce path.
"""

import time

import torch
import torch.distributed as dist

from . import ccube


def measure_peer_bandwidth(pg=None, nbytes: int = 64 << 20, reps: int = 3):
    """bw[i][j] in GB/s for rank i -> rank j, identical on every rank.

    On GPUs (an NCCL group) this is the library's own store path
    (``ccube_measure_peer_bandwidth``: the AllReduce kernel's 128-bit loads from
    local HBM and stores into the peer's HBM, device-timed after a device-side
    barrier, every rank storing to its k-th successor at once) through a temporary
    identity-placed communicator — the bandwidth the tree edges will actually see.
    On CPU (gloo, the host tests) it falls back to timing send/recv per ordered pair."""
    pg = pg or dist.group.WORLD
    P, me = dist.get_world_size(pg), dist.get_rank(pg)
    on_gpu = dist.get_backend(pg) == "nccl"
    if on_gpu:
        ccube.set_placement(None)
        ccube.init_distributed(pg, tree="single")
        try:
            pair, _ = ccube.measure_peer_bandwidth(nbytes, reps)
        finally:
            ccube.finalize()
        return pair
    buf = torch.empty(nbytes // 4, dtype=torch.float32)
    bw = torch.zeros(P, P, dtype=torch.float64)
    for i in range(P):
        for j in range(P):
            if i == j:
                continue
            dist.barrier(group=pg)
            best = float("inf")
            for _ in range(reps):
                t0 = time.perf_counter()
                if me == i:
                    dist.send(buf, dst=dist.get_global_rank(pg, j), group=pg)
                elif me == j:
                    dist.recv(buf, src=dist.get_global_rank(pg, i), group=pg)
                best = min(best, time.perf_counter() - t0)
            if me == j:
                bw[i, j] = nbytes / best / 1e9
    # the receiver's number is authoritative; share it with everyone
    dist.all_reduce(bw, op=dist.ReduceOp.SUM, group=pg)
    return bw.tolist()


def plan(pg=None, kind: str = "double", **measure_kw):
    """Measure, plan and return the placement (the same list on every rank)."""
    bw = measure_peer_bandwidth(pg, **measure_kw)
    for i in range(len(bw)):
        bw[i][i] = 1.0   # unused (no tree edge joins a rank to itself)
    return ccube.plan_placement(bw, kind), bw

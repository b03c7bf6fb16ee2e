"""Placement (reading R19, the NVSwitch form of §IV's detour routes):
the oracle's definition and planner pinned by hand-derived cases and brute force,
then the library's host-side planner and placed trees checked against it, and the
multi-process agreement check over gloo.  No GPU needed."""

import itertools
import os
import socket

import numpy as np
import pytest

from oracle import allreduce as oar
from oracle import placement as opl
from oracle import trees as otrees
from paper_conf_hpca_sanghoonsk23_b200 import ccube


# ---- oracle ------------------------------------------------------------------
def test_placed_tree_relabels_positions():
    """perm = reversal at P=4: tree 0 (0 <- 2 <- {1, 3}) becomes 3 <- 1 <- {0, 2}."""
    t = otrees.placed(otrees.tree0(4), [3, 2, 1, 0])
    assert t.root == 3
    assert t.parent == (1, 3, 1, -1)
    assert t.children[1] == (0, 2)           # ascending rank: the combine order (R2)


def test_placed_order_pin_fp32():
    """Hand-derived: identity gives x0 + ((x2 + x1) + x3); the reversal gives
    x3 + ((x1 + x0) + x2).  With x = (1, 2^24, 1, -2^24): identity 1.0 (P:L119's
    tree), reversal fl(2^24 + 1) = 2^24 (tie to even), + 1 -> 2^24, -2^24 -> 0.0."""
    xs = [np.array([v], np.float32) for v in (1.0, 2.0 ** 24, 1.0, -2.0 ** 24)]
    assert oar.reference(xs, "single", 16, "float32")[0][0] == 1.0
    assert oar.reference(xs, "single", 16, "float32", perm=[3, 2, 1, 0])[0][0] == 0.0


@pytest.mark.parametrize("kind", ["single", "double", "rotated"])
def test_placed_int32_is_the_plain_sum(kind):
    rng = np.random.default_rng(3)
    xs = [rng.integers(-2 ** 31, 2 ** 31, 300, dtype=np.int64).astype(np.int32) for _ in range(5)]
    want = np.sum(np.stack(xs).astype(np.int64), axis=0).astype(np.uint64).astype(np.uint32)
    for perm in ([4, 3, 2, 1, 0], [2, 0, 4, 1, 3]):
        out, _ = oar.replay(xs, kind, 64, "int32", perm=perm)
        for o in out:
            assert np.array_equal(o.view(np.uint32), want)


@pytest.mark.parametrize("kind", ["single", "double", "rotated"])
def test_replay_equals_reference_with_placement(kind):
    rng = np.random.default_rng(4)
    xs = [rng.standard_normal(777).astype(np.float32) for _ in range(6)]
    perm = [5, 1, 3, 0, 2, 4]
    ref = oar.reference(xs, kind, 128, "float32", perm=perm)[0]
    out, _ = oar.replay(xs, kind, 128, "float32", perm=perm)
    for o in out:
        assert np.array_equal(o, ref)


def test_plan_uniform_is_identity():
    for P in range(1, 7):
        assert opl.plan(P, "double", np.full((P, P), 7.0)) == list(range(P))


def test_plan_avoids_a_slow_pair():
    """P=4 single tree uses pairs {0,2}, {1,2}, {2,3}; making 0<->2 slow forces a
    placement in which ranks 0 and 2 are not adjacent in the tree."""
    bw = np.full((4, 4), 100.0)
    bw[0, 2] = bw[2, 0] = 10.0
    perm = opl.plan(4, "single", bw)
    t = otrees.trees(4, "single", perm)[0]
    assert t.parent[0] != 2 and t.parent[2] != 0
    assert opl.cost(4, "single", bw, perm) == pytest.approx(1 / 100)


def test_plan_detour_matrix_no_path():
    """bw <= 0 = no direct path (the DGX-1 cube mesh's missing pairs): the plan
    uses only existing pairs when a placement with finite cost exists."""
    P = 4
    bw = np.full((P, P), 50.0)
    bw[0, 1] = bw[1, 0] = 0.0
    bw[0, 3] = bw[3, 0] = 0.0
    perm = opl.plan(P, "single", bw)
    assert np.isfinite(opl.cost(P, "single", bw, perm))


@pytest.mark.parametrize("P", [3, 4, 5])
@pytest.mark.parametrize("kind", ["single", "double", "rotated"])
def test_plan_is_the_brute_force_minimum(P, kind):
    """plan() (relabelled loads) vs the definition (cost() rebuilds the placed trees)."""
    rng = np.random.default_rng(P * 10 + len(kind))
    bw = rng.uniform(10, 100, (P, P))
    best = min(opl.cost(P, kind, bw, p) for p in itertools.permutations(range(P)))
    assert opl.cost(P, kind, bw, opl.plan(P, kind, bw)) == pytest.approx(best)


# ---- library (host-only functions) --------------------------------------------
@pytest.mark.parametrize("P", [2, 3, 4, 5, 6, 7, 8])
@pytest.mark.parametrize("kind", ["single", "double", "rotated"])
def test_library_placed_trees_match_oracle(P, kind):
    rng = np.random.default_rng(P)
    perm = [int(v) for v in rng.permutation(P)]
    for t, tree in enumerate(otrees.trees(P, kind, perm)):
        assert ccube.tree_parents_placed(P, kind, t, perm) == list(tree.parent)
    assert ccube.tree_parents_placed(P, kind, 0, None) == ccube.tree_parents(P, kind, 0)


@pytest.mark.parametrize("P", [2, 4, 6, 8])
@pytest.mark.parametrize("kind", ["single", "double", "rotated"])
def test_library_plan_matches_oracle(P, kind):
    rng = np.random.default_rng(100 + P)
    for _ in range(3):
        bw = rng.uniform(20, 100, (P, P)).round(1)
        assert ccube.plan_placement(bw, kind) == opl.plan(P, kind, bw)
    assert ccube.plan_placement(np.full((P, P), 3.0), kind) == list(range(P))


def test_library_placement_validation():
    for bad in ([0, 0, 1], [0, 1, 3], [-1, 0, 1]):
        with pytest.raises(ccube.CCubeError) as e:
            ccube.set_placement(bad)
        assert e.value.code == ccube.ERR_INVALID_ARG
    with pytest.raises(ccube.CCubeError) as e:
        ccube.tree_parents_placed(3, "single", 0, [0, 2, 2])
    assert e.value.code == ccube.ERR_INVALID_ARG
    with pytest.raises(ccube.CCubeError) as e:
        ccube.plan_placement(np.ones((9, 9)), "single")
    assert e.value.code in (ccube.ERR_INVALID_ARG, ccube.ERR_UNSUPPORTED)
    # a placement for 3 ranks does not fit a 4-rank init
    ccube.set_placement([2, 1, 0])
    try:
        with pytest.raises(ccube.CCubeError) as e:
            ccube.init(4)
        assert e.value.code == ccube.ERR_INVALID_ARG
    finally:
        ccube.set_placement(None)


# ---- multi-process agreement (gloo, world size 2) ------------------------------
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, perms, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_hpca_sanghoonsk23_b200 import ccube as cc
    try:
        cc.set_placement(perms[rank])
        cc.init(world, rank=rank, nlocal=1, device=0, tree="double", pg=dist.group.WORLD)
        q.put((rank, 0, ""))
        cc.finalize()
    except cc.CCubeError as e:
        q.put((rank, e.code, str(e)))
    dist.destroy_process_group()


def _run(perms):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, perms, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = sorted(q.get(timeout=120) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    return out


def test_gloo_placement_agreement_ws2():
    for rank, code, msg in _run([[1, 0], [1, 0]]):
        assert code in (ccube.SUCCESS, ccube.ERR_CUDA, ccube.ERR_UNSUPPORTED), msg
        assert "disagree" not in msg


def test_gloo_placement_mismatch_ws2():
    for rank, code, msg in _run([[1, 0], None]):
        assert code == ccube.ERR_INVALID_ARG, msg
        assert "disagree" in msg


def _measure_worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_hpca_sanghoonsk23_b200 import placement
    perm, bw = placement.plan(kind="single", nbytes=1 << 16, reps=1)
    q.put((rank, perm, bw))
    dist.destroy_process_group()


def test_gloo_measure_and_plan_ws3():
    """The init-time helper over gloo (world size 3): every rank gets the same
    bandwidth matrix (positive off the diagonal) and the same placement."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_measure_worker, args=(r, 3, port, q)) for r in range(3)]
    for p in procs:
        p.start()
    out = sorted(q.get(timeout=120) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    perms = [o[1] for o in out]
    bws = [o[2] for o in out]
    assert perms[0] == perms[1] == perms[2] and sorted(perms[0]) == [0, 1, 2]
    assert bws[0] == bws[1] == bws[2]
    assert all(bws[0][i][j] > 0 for i in range(3) for j in range(3) if i != j)

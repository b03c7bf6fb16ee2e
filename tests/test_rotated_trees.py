"""The rotated multi-tree set (reading R17): P trees, tree t = tree 0
with ranks renamed (v + t) mod P, chunk c on tree c mod P.  Pins: structure
(spanning, every rank in every position once), the closed-form port load
2(P-1)/P, brute-force int32 sums, a hand-derived fp32 order pin, the gate's
per-tree chunk counts, and the library's tree builder against the oracle's."""

import math

import numpy as np
import pytest

from oracle import allreduce, costmodel, gradq, partition, trees
from paper_conf_hpca_sanghoonsk23_b200 import inputs


def _position(tree, v):
    """(depth, index among siblings by tree-0 rank) — v's position in the shape."""
    d, u = 0, v
    while tree.parent[u] != -1:
        u = tree.parent[u]
        d += 1
    return d, len(tree.children[v])


@pytest.mark.parametrize("P", range(1, 9))
def test_structure(P):
    ts = trees.trees(P, "rotated")
    assert len(ts) == P
    t0 = trees.tree0(P)
    for t, tr in enumerate(ts):
        assert tr.root == t
        assert sum(len(c) for c in tr.children) == P - 1
        for v in range(P):
            # the renaming maps tree 0's position of u to rank (u + t) mod P
            u = (v - t) % P
            assert _position(tr, v) == _position(t0, u)
            assert list(tr.children[v]) == sorted(tr.children[v])
    # every rank holds every position exactly once over the set
    for v in range(P):
        roles = sorted(_position(ts[t], v) for t in range(P))
        assert roles == sorted(_position(t0, u) for u in range(P))


@pytest.mark.parametrize("P", range(2, 9))
def test_port_load_is_bandwidth_optimal(P):
    """Each rank sends (#children + [not root]) * N/P per tree: summed over the set,
    exactly 2(P-1)/P * N for EVERY rank — the ring's per-rank load."""
    loads = costmodel.port_loads(P, "rotated", 1.0)
    for x in loads:
        assert math.isclose(x, 2 * (P - 1) / P)
    assert math.isclose(costmodel.busbw_ceiling(P, "rotated", 900), 900.0)
    assert max(costmodel.port_loads(8, "double", 1.0)) == 2.0   # vs 1.75 here


@pytest.mark.parametrize("P", range(1, 9))
@pytest.mark.parametrize("full_range", [False, True])
def test_int32_equals_bruteforce_sum(P, full_range):
    count = 3001
    xs = [inputs.gradients(r, count, "int32", seed=11, full_range=full_range) for r in range(P)]
    out = allreduce.reference(xs, "rotated", 1024, "int32")
    s = np.zeros(count, dtype=np.int64)
    for x in xs:
        s += x.astype(np.int64)
    want = ((s + 2 ** 31) % 2 ** 32 - 2 ** 31).astype(np.int32)
    for o in out:
        assert np.array_equal(o, want)


def test_order_pin_P4(golden):
    """Chunk 1 travels on tree 1 (root 1 <- 3 <- {0, 2}): x1 + ((x3 + x0) + x2)."""
    g = golden("order_pins.txt")
    vals = [float(v) for v in g["rotated_order_pin_inputs"]]
    xs = []
    for r in range(4):
        x = np.zeros(8, dtype=np.float32)
        x[0] = x[4] = vals[r]          # element 0 in chunk 0 (tree 0), element 4 in chunk 1
        xs.append(x)
    out = allreduce.reference(xs, "rotated", 16, "float32")
    assert out[0][4] == float(g["rotated_tree1_result"][0])
    assert out[0][0] == float(g["rotated_tree0_result"][0])
    assert partition.tree_of_chunk(1, 4) == 1


@pytest.mark.parametrize("P", [2, 3, 5, 8])
@pytest.mark.parametrize("dtype", ["float32", "bfloat16"])
@pytest.mark.parametrize("overlap", [True, False])
def test_replay_equals_definition(P, dtype, overlap):
    count = 2600 + P
    xs = [inputs.gradients(r, count, dtype, seed=3) for r in range(P)]
    ref = allreduce.reference(xs, "rotated", 1024, dtype)
    out, scheds = allreduce.replay(xs, "rotated", 1024, dtype, overlap=overlap)
    assert len(scheds) == P
    for r in range(P):
        assert np.array_equal(out[r], ref[0])


def test_need_per_tree_counts():
    assert gradq.need_per_tree(7, 8) == [1, 1, 1, 1, 1, 1, 1, 0]
    assert gradq.need_per_tree(10, 4) == [3, 3, 2, 2]
    assert gradq.need_per_tree(0, 3) == [0, 0, 0]
    for lct in range(40):
        for T in range(1, 9):
            n = gradq.need_per_tree(lct, T)
            assert sum(n) == lct
            assert max(n) - min(n) <= 1


@pytest.mark.parametrize("P", range(1, 9))
def test_library_builder_matches_oracle(P):
    from paper_conf_hpca_sanghoonsk23_b200 import ccube
    for t in range(P):
        assert ccube.tree_parents(P, "rotated", t) == list(trees.trees(P, "rotated")[t].parent)
    with pytest.raises(ccube.CCubeError):
        ccube.tree_parents(P, "rotated", P)

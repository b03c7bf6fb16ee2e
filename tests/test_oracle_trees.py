"""Pins for oracle.trees (a1).  Paper: P:L119 worked tree, fn4 P:L153 flipped tree."""

import pytest

from oracle import trees


def _reaches_root(t, v):
    seen = set()
    while t.parent[v] != -1:
        if v in seen:
            return False
        seen.add(v)
        v = t.parent[v]
    return v == t.root


@pytest.mark.parametrize("P", range(1, 17))
@pytest.mark.parametrize("kind", ["single", "double"])
def test_spanning_binary_trees(P, kind):
    for t in trees.trees(P, kind):
        assert sorted(range(P)) == sorted(set(range(P)))
        assert sum(1 for v in range(P) if t.parent[v] == -1) == 1
        for v in range(P):
            assert _reaches_root(t, v)
            assert len(t.children[v]) <= 2
            assert list(t.children[v]) == sorted(t.children[v])
            for c in t.children[v]:
                assert t.parent[c] == v
        # edges = P - 1
        assert sum(len(c) for c in t.children) == P - 1


@pytest.mark.parametrize("P", range(2, 17))
def test_root_has_single_child_and_log_depth(P):
    t = trees.tree0(P)
    assert t.root == 0
    assert len(t.children[0]) == 1
    # the root's child is the largest power of two below P
    assert t.children[0][0] == 1 << ((P - 1).bit_length() - 1)
    # depth = ceil(log2 P): the paper's "depth of the tree is proportional to log(P)"
    assert t.depth() == (P - 1).bit_length()


def test_worked_example_tree_P4(golden):
    """root N4 <- N2 <- {N1, N3}  ==  0 <- 2 <- {1, 3} (golden fig5_schedule.txt)."""
    g = golden("fig5_schedule.txt")
    t = trees.tree0(4)
    assert list(t.parent) == [int(x) for x in g["tree_parent"]]
    assert t.children[2] == (1, 3)


@pytest.mark.parametrize("P", [2, 4, 8, 16])
def test_flip_inverts_nodes_and_leaves(P):
    """fn4 P:L153: 'the first tree is flipped to invert the nodes and leaves'.
    For power-of-two P every tree-0 leaf is a tree-1 interior node, and only the
    two roots (0 and P-1, each with one child) are non-leaves in both."""
    t0, t1 = trees.tree0(P), trees.tree1(P)
    assert set(t0.leaves()) == set(t1.interior())
    assert set(t1.leaves()) == set(t0.interior())
    # every rank is an interior non-root in at most one tree
    for v in range(P):
        inner = [v != t.root and len(t.children[v]) > 0 for t in (t0, t1)]
        assert sum(inner) <= 1


def test_P8_tables():
    t0, t1 = trees.tree0(8), trees.tree1(8)
    assert t0.children[0] == (4,) and t0.children[4] == (2, 6)
    assert t0.children[2] == (1, 3) and t0.children[6] == (5, 7)
    assert t1.root == 7 and t1.children[7] == (3,) and t1.children[3] == (1, 5)
    assert t1.children[1] == (0, 2) and t1.children[5] == (4, 6)
    assert set(t0.leaves()) == {1, 3, 5, 7}
    assert set(t1.leaves()) == {0, 2, 4, 6}


@pytest.mark.parametrize("P", [3, 5, 7])
def test_odd_shift_keeps_roots_apart(P):
    t0, t1 = trees.tree0(P), trees.tree1(P)
    assert t0.root != t1.root
    assert t1.root == 1


@pytest.mark.parametrize("P", range(2, 17))
def test_parent_rule_matches_children_rule(P):
    """Second description of the same tree: children of r with lowest
    set bit b are r - b/2 and r + b/2, halving the right offset until in range."""
    t = trees.tree0(P)
    for r in range(1, P):
        b = r & -r
        kids = []
        if b > 1:
            kids.append(r - b // 2)
            off = b // 2
            while off and r + off >= P:
                off //= 2
            if off:
                kids.append(r + off)
        assert tuple(sorted(kids)) == t.children[r], (P, r)

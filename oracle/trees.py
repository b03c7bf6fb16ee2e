"""a1 — logical tree construction (oracle; test infrastructure only).

Paper basis
  * Tree AllReduce: "reduction as data moves up the tree and broadcast as data
    moves down the tree"; the 4-node worked example has root N4 <- N2 <- {N1, N3}
    (§III-A, Fig 5(a)).
  * Double binary tree [45]: "a double binary tree ... is commonly used with two
    trees" (§III-B) and "the first tree is flipped to invert the nodes and
    leaves to create the second tree" (fn4).

Reading R1: tree 0 is the binary tree rooted at rank 0 with a
single child; every other rank r with lowest set bit b has parent
``(r ^ b) | (b << 1)`` or, if that is >= P, ``r ^ b``.  At P=4 this is exactly the
paper's example 0 <- 2 <- {1, 3} (ranks = N_i - 1 with N4 the root relabelled 0).
Tree 1 relabels tree 0 by phi(v) = P-1-v for even P (the "flip": tree-0 leaves
become tree-1 interior nodes) and phi(v) = (v+1) mod P for odd P.
Children are listed in ascending rank; that order is the combine order (R2).

Rotated set (reading R17): the NVSwitch form of §IV's
topology-aware trees — P trees, tree t = tree 0 with every rank v
renamed (v + t) mod P, so every rank holds every tree position exactly once and
each rank's port carries 2(P-1)/P of the buffer per direction.

Placement (reading R19): the NVSwitch form of §IV's detour routes is
the choice of which physical rank hosts which tree position.  A placement is a
permutation perm: position v of every tree of the kind is hosted by rank
perm[v]; children are re-listed in ascending (physical) rank, which is the
combine order (R2), so a placement can change fp results (not int32 ones).
Identity = the trees above.
"""

from dataclasses import dataclass
from typing import List, Optional, Sequence, Tuple


@dataclass(frozen=True)
class Tree:
    P: int
    root: int
    parent: Tuple[int, ...]                 # parent[v], -1 at the root
    children: Tuple[Tuple[int, ...], ...]   # children[v], ascending rank

    def depth(self) -> int:
        """Depth in edges = max over v of the path length to the root."""
        best = 0
        for v in range(self.P):
            d, u = 0, v
            while self.parent[u] != -1:
                u = self.parent[u]
                d += 1
            best = max(best, d)
        return best

    def leaves(self) -> List[int]:
        return [v for v in range(self.P) if not self.children[v]]

    def interior(self) -> List[int]:
        """Ranks with at least one child (the root included)."""
        return [v for v in range(self.P) if self.children[v]]


def _lowest_set_bit(r: int) -> int:
    return r & -r


def btree_parent(r: int, P: int) -> int:
    """Parent of rank r in tree 0 (R1).  Rank 0 is the root."""
    if r == 0:
        return -1
    b = _lowest_set_bit(r)
    up = (r ^ b) | (b << 1)
    return up if up < P else (r ^ b)


def _from_parent(P: int, parent: List[int]) -> Tree:
    children: List[List[int]] = [[] for _ in range(P)]
    root = -1
    for v in range(P):
        if parent[v] == -1:
            root = v
        else:
            children[parent[v]].append(v)
    return Tree(P=P, root=root, parent=tuple(parent),
                children=tuple(tuple(sorted(c)) for c in children))


def tree0(P: int) -> Tree:
    """The single (first) binary tree, rooted at rank 0."""
    if P < 1:
        raise ValueError("P must be >= 1")
    return _from_parent(P, [btree_parent(r, P) for r in range(P)])


def relabel(P: int, v: int) -> int:
    """phi: tree-0 position v -> rank in tree 1 (R1; fn4 P:L153)."""
    if P % 2 == 0:
        return P - 1 - v
    return (v + 1) % P


def tree1(P: int) -> Tree:
    """The second tree of the double tree: tree 0 with every rank v renamed phi(v)."""
    t0 = tree0(P)
    parent = [-1] * P
    for v in range(P):
        pv = t0.parent[v]
        parent[relabel(P, v)] = -1 if pv == -1 else relabel(P, pv)
    return _from_parent(P, parent)


def rotated(P: int, t: int) -> Tree:
    """Tree t of the rotated set (R17): tree 0 with every rank v renamed (v + t) mod P."""
    t0 = tree0(P)
    parent = [-1] * P
    for v in range(P):
        pv = t0.parent[v]
        parent[(v + t) % P] = -1 if pv == -1 else (pv + t) % P
    return _from_parent(P, parent)


def placed(tree: Tree, perm: Sequence[int]) -> Tree:
    """R19: the tree with position v hosted by rank perm[v] (children re-sorted)."""
    P = tree.P
    if sorted(perm) != list(range(P)):
        raise ValueError(f"placement {list(perm)} is not a permutation of 0..{P - 1}")
    parent = [-1] * P
    for v in range(P):
        pv = tree.parent[v]
        parent[perm[v]] = -1 if pv == -1 else perm[pv]
    return _from_parent(P, parent)


def trees(P: int, kind: str, perm: Optional[Sequence[int]] = None) -> List[Tree]:
    """kind = 'single' -> [tree0]; 'double' -> [tree0, tree1]; 'rotated' -> P trees;
    each placed by ``perm`` (R19) when given."""
    if kind == "single":
        ts = [tree0(P)]
    elif kind == "double":
        ts = [tree0(P), tree1(P)]
    elif kind == "rotated":
        ts = [rotated(P, t) for t in range(max(P, 1))]
    else:
        raise ValueError(kind)
    return ts if perm is None else [placed(t, perm) for t in ts]

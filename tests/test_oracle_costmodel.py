"""Pins for oracle.costmodel: eqs 1-7 re-derived, port loads against the ring total."""

import math

import pytest

from oracle import costmodel, trees


A, B, N = 2e-6, 1 / 900e9, 64 * 2 ** 20


@pytest.mark.parametrize("P", [2, 4, 8, 16])
def test_eq6_is_eq3_at_eq4(P):
    """substituting K_opt (eq 4) into 2 x eq 3 gives eq 6 exactly."""
    k = costmodel.k_opt(P, N, A, B)
    assert math.isclose(2 * costmodel.t_phase(P, N, k, A, B), costmodel.t_tree(P, N, A, B), rel_tol=1e-12)


@pytest.mark.parametrize("P", [2, 4, 8, 16])
def test_eq4_minimises_eq3(P):
    k = costmodel.k_opt(P, N, A, B)
    t = costmodel.t_phase(P, N, k, A, B)
    for f in (0.5, 0.9, 1.1, 2.0):
        assert costmodel.t_phase(P, N, k * f, A, B) > t


@pytest.mark.parametrize("P", [2, 4, 8, 16])
def test_eq7_reading(P):
    """R7: the optimum of (2 log P + K)(alpha + beta N/K) has coefficient 2*sqrt(2),
    not eq 7's 3; eq 7 over-estimates by (3 - 2 sqrt 2) sqrt(alpha beta N log P)."""
    L = math.log2(P)
    kstar = math.sqrt(2 * L * B * N / A)
    exact = costmodel.t_c1_steps(P, N, kstar, A, B)
    assert math.isclose(exact, costmodel.t_c1_exact(P, N, A, B), rel_tol=1e-12)
    gap = costmodel.t_c1_eq7(P, N, A, B) - exact
    assert math.isclose(gap, (3 - 2 * math.sqrt(2)) * math.sqrt(A * B * N * L), rel_tol=1e-9)


def test_eq1_eq2():
    assert math.isclose(costmodel.t_ring(8, N, A, B), 2 * costmodel.t_allgather(8, N, A, B))


@pytest.mark.parametrize("P", range(2, 17))
@pytest.mark.parametrize("kind", ["single", "double"])
def test_port_loads_total_equals_ring(P, kind):
    """Any spanning tree moves 2(P-1) N bytes over all ranks (P-1 edges, N up + N
    down each) — the same total as a ring's 2(P-1)/P N per rank (eq 2)."""
    loads = costmodel.port_loads(P, kind, 1.0)
    assert math.isclose(sum(loads), 2 * (P - 1))


def test_port_ceiling_table():
    """SURVEY §8(d) ceilings at 900 GB/s."""
    assert math.isclose(costmodel.busbw_ceiling(8, "single", 900), 525.0)
    assert math.isclose(costmodel.busbw_ceiling(8, "double", 900), 787.5)
    assert math.isclose(costmodel.busbw_ceiling(4, "double", 900), 675.0)
    assert math.isclose(costmodel.busbw_ceiling(2, "single", 900), 900.0)
    assert max(costmodel.port_loads(8, "single", 1.0)) == 3
    t0 = trees.tree0(8)
    assert costmodel.port_loads(8, "single", 1.0)[0] == len(t0.children[0])


@pytest.mark.parametrize("P", [2, 3, 4, 5, 8, 16])
def test_ring_beta_term_is_the_bandwidth_optimal_port_load(P):
    """Eq 2's bandwidth term 2((P-1)/P) beta N is the per-rank load of a ring; it must
    equal, independently, the per-rank port load of the rotated tree set computed
    from the trees (every rank holds every position once, R17) — and lower-bound
    every tree shape's busiest port."""
    ring_beta = costmodel.t_ring(P, N, 0.0, B) / B          # alpha = 0: bytes per rank
    rot = costmodel.port_loads(P, "rotated", N)
    assert all(math.isclose(x, ring_beta) for x in rot)
    for kind in ("single", "double"):
        assert max(costmodel.port_loads(P, kind, N)) >= ring_beta * (1 - 1e-12)


@pytest.mark.parametrize("P", [2, 4, 8])
def test_allgather_is_the_ring_half(P):
    """Eq 1 vs eq 2 at any P: the ring AllReduce is a reduce-scatter plus an
    all-gather of P-1 steps each, so t_ring = 2 t_allgather for every (alpha, beta);
    with beta = 0 it is 2(P-1) alpha (P-1 dependent steps per phase)."""
    assert math.isclose(costmodel.t_ring(P, N, A, B), 2 * costmodel.t_allgather(P, N, A, B))
    assert math.isclose(costmodel.t_ring(P, N, A, 0.0), 2 * (P - 1) * A)
    assert math.isclose(costmodel.t_allgather(P, N, 0.0, B), (P - 1) / P * N * B)

"""Pins for oracle.schedule: the paper's worked schedule (Fig 5) and closed forms."""

import pytest

from oracle import schedule, trees


def test_fig5_worked_schedule(golden):
    g = golden("fig5_schedule.txt")
    P, K = int(g["P"][0]), int(g["K"][0])
    t = trees.tree0(P)
    b = schedule.simulate(t, K, overlap=False)
    c1 = schedule.simulate(t, K, overlap=True)
    assert b.total_steps == int(g["baseline_total_steps"][0])          # P:L119 "Step 10"
    assert c1.total_steps == int(g["overlap_total_steps"][0])          # P:L163 "7 steps"
    assert max(b.final) == int(g["baseline_reduction_complete_at_root_step"][0])
    assert b.final[0] == int(g["chunk1_fully_reduced_step"][0])       # P:L127 "Step 2"
    assert c1.down_send[t.root][0] == int(g["overlap_chunk1_broadcast_begins_step"][0])
    # in Step 7 the root sends chunk 2 while N2 (rank 2) sends chunk 1
    assert b.down_send[t.root].index(7) + 1 == int(g["baseline_step7_root_sends_chunk"][0])
    assert b.down_send[2].index(7) + 1 == int(g["baseline_step7_rank2_sends_chunk"][0])


@pytest.mark.parametrize("P", range(2, 17))
@pytest.mark.parametrize("K", [1, 2, 4, 16, 390])
def test_closed_forms(P, K):
    """By induction on node height: a node of height h sends chunk k up at k+1+h, so
    final[k] = k + D; B: 2(K + D - 1) steps, C1: K + 2D - 1 steps (the paper's
    2(log P + K) and 2 log P + K, up to the constant); turnaround B: K+2D-1,
    C1: 2D."""
    t = trees.tree0(P)
    D = t.depth()
    b = schedule.simulate(t, K, overlap=False)
    c1 = schedule.simulate(t, K, overlap=True)
    assert b.total_steps == 2 * (K + D - 1)
    assert c1.total_steps == K + 2 * D - 1
    assert b.turnaround == K + 2 * D - 1
    assert c1.turnaround == 2 * D
    assert b.final == c1.final == [k + D for k in range(K)]


@pytest.mark.parametrize("P", [2, 3, 4, 5, 8])
@pytest.mark.parametrize("overlap", [True, False])
def test_in_order_landing(P, overlap):
    """Obs #3 and P:L193: every rank receives chunks in order."""
    for t in trees.trees(P, "double"):
        s = schedule.simulate(t, 9, overlap)
        for v in range(P):
            assert all(a < b for a, b in zip(s.land[v], s.land[v][1:]))


def test_appendix_turnaround_table():
    """SURVEY App. A step-model table (P=8: K=16 -> 36/21 steps, turnaround 21 vs 6)."""
    t = trees.tree0(8)
    for K, bsteps, csteps, tb, tc in [(16, 36, 21, 21, 6), (256, 516, 261, 261, 6), (390, 784, 395, 395, 6)]:
        b = schedule.simulate(t, K, False)
        c = schedule.simulate(t, K, True)
        assert (b.total_steps, c.total_steps, b.turnaround, c.turnaround) == (bsteps, csteps, tb, tc)


def test_P1_and_K0_degenerate():
    s = schedule.simulate(trees.tree0(1), 5, True)
    assert s.total_steps == 0
    s = schedule.simulate(trees.tree0(4), 0, True)
    assert s.total_steps == 0 and s.events() == []


def test_overlap_never_slower():
    for P in range(2, 9):
        for K in (1, 3, 10):
            t = trees.tree0(P)
            assert schedule.simulate(t, K, True).total_steps <= schedule.simulate(t, K, False).total_steps

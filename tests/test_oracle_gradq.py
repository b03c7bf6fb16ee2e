"""Pins for oracle.gradq: Fig 8 Layer-Chunk Table, Fig 11 semaphore semantics, gates."""

import numpy as np
import pytest

from oracle import gradq, schedule, trees


def test_fig8_layer_chunk_table(golden):
    g = golden("fig8_lct.txt")
    per_layer = [int(v) for v in g["chunks_per_layer"]]
    E = 1000
    ends, acc = [], 0
    for n in per_layer:
        acc += n * E
        ends.append(acc)
    assert gradq.layer_chunk_table(ends, E) == [int(v) for v in g["lct"]]


def test_lct_straddling_chunk_gates_both_layers():
    """R10: a chunk holding elements of two layers is needed by both."""
    assert gradq.layer_chunk_table([10, 15, 40], 10) == [1, 2, 4]
    assert gradq.layer_chunk_table([0, 0, 5], 10) == [0, 0, 1]
    with pytest.raises(ValueError):
        gradq.layer_chunk_table([10, 5], 10)


def test_need_per_tree():
    assert gradq.need_per_tree(5, 1) == [5]
    assert gradq.need_per_tree(5, 2) == [3, 2]
    assert gradq.need_per_tree(1, 2) == [1, 0]
    assert gradq.need_per_tree(0, 2) == [0, 0]


def test_fig11_semaphore_semantics():
    s = gradq.Semaphore()
    assert not s.can_wait()            # wait: spin while cnt == 0
    assert s.check(0) and not s.check(1)
    s.post(2)
    s.post(2)
    assert not s.can_post(2)           # post: spin while cnt == value
    with pytest.raises(RuntimeError):
        s.post(2)
    assert s.check(2)                  # check: spin while cnt < value; no change
    assert s.cnt == 2
    s.wait()
    assert s.cnt == 1


@pytest.mark.parametrize("P", [2, 4, 8])
@pytest.mark.parametrize("kind", ["single", "double"])
@pytest.mark.parametrize("overlap", [True, False])
def test_gate_opens_at_landing_of_last_needed_chunk(P, kind, overlap):
    """a layer starts once the semaphore >= LCT[l]; with in-order landing
    this is exactly the landing step of the layer's last chunk (per tree, maxed)."""
    K = 15
    ts = trees.trees(P, kind)
    ids = [[c for c in range(K) if (c % len(ts)) == t] for t in range(len(ts))]
    scheds = [schedule.simulate(tr, len(ids[t]), overlap) for t, tr in enumerate(ts)]
    lct = [1, 3, 6, 10, 15]
    for v in range(P):
        gates = gradq.gate_steps([s.land[v] for s in scheds], lct)
        for l, n in enumerate(lct):
            need = gradq.need_per_tree(n, len(ts))
            want = max(scheds[t].land[v][need[t] - 1] for t in range(len(ts)) if need[t] > 0)
            assert gates[l] == want
        assert gates == sorted(gates)


def test_chaining_gates_open_earlier_with_overlap():
    """C1 shortens gradient turnaround: every gate opens no later than in B."""
    t = trees.tree0(8)
    b = schedule.simulate(t, 20, False)
    c = schedule.simulate(t, 20, True)
    lct = [2, 5, 9, 14, 20]
    for v in range(8):
        gb = gradq.gate_steps([b.land[v]], lct)
        gc = gradq.gate_steps([c.land[v]], lct)
        assert all(x <= y for x, y in zip(gc, gb))


def test_forward_timeline_model():
    gates = [1, 3, 6, 10, 15]
    compute = [4, 3, 2, 1, 1]
    chained = gradq.forward_timeline(gates, compute, True, comm_end=15)
    unchained = gradq.forward_timeline(gates, compute, False, comm_end=15)
    assert chained == [5, 8, 10, 11, 16]
    assert unchained == [19, 22, 24, 25, 26]
    assert chained[-1] <= unchained[-1]


def test_sgd_update_closed_forms():
    """R18: w - alpha * g elementwise; exact cases."""
    w = np.array([1.0, -2.0, 3.5, 0.0], dtype=np.float32)
    g = np.array([2.0, 4.0, -1.0, 0.0], dtype=np.float32)
    assert np.array_equal(gradq.sgd_update(w, g, 0.5), np.array([0.0, -4.0, 4.0, 0.0], np.float32))
    assert np.array_equal(gradq.sgd_update(w, g, 0.0), w)
    assert gradq.sgd_update(w, g, 0.5).dtype == np.float32


def test_sgd_update_rounds_twice_no_fma(golden):
    """R18 pin: the product is rounded before the subtraction (an FMA differs)."""
    gl = golden("order_pins.txt")
    w, g, a = (float(v) for v in gl["sgd_no_fma_pin_w_g_alpha"])
    got = gradq.sgd_update(np.array([w], np.float32), np.array([g], np.float32), a)[0]
    assert got == float(gl["sgd_no_fma_pin_result"][0])
    exact = w - a * g          # python floats are binary64: exact here
    assert exact == float(gl["sgd_fma_result"][0])
    assert np.float32(exact) != got

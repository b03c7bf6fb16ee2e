"""Pins for oracle.allreduce: brute force, closed forms, worked inputs, invariants."""

import numpy as np
import pytest

from oracle import allreduce, arith, partition, trees
from paper_conf_hpca_sanghoonsk23_b200 import inputs

CB = 1024  # small chunks so tiny buffers still span several chunks


def _xs(P, count, dtype, seed=7, full_range=False):
    return [inputs.gradients(r, count, dtype, seed=seed, full_range=full_range) for r in range(P)]


@pytest.mark.parametrize("P", range(1, 9))
@pytest.mark.parametrize("kind", ["single", "double"])
@pytest.mark.parametrize("full_range", [False, True])
def test_int32_equals_bruteforce_sum_mod_2_32(P, kind, full_range):
    xs = _xs(P, 3001, "int32", full_range=full_range)
    out = allreduce.reference(xs, kind, CB, "int32")
    s = np.zeros(3001, dtype=np.int64)
    for x in xs:
        s += x.astype(np.int64)
    want = ((s + 2 ** 31) % 2 ** 32 - 2 ** 31).astype(np.int32)
    for o in out:
        assert np.array_equal(o, want)


@pytest.mark.parametrize("dtype", arith.DTYPES)
def test_P1_identity(dtype):
    xs = _xs(1, 777, dtype)
    for kind in ("single", "double"):
        assert np.array_equal(allreduce.reference(xs, kind, CB, dtype)[0], xs[0])


def test_P2_is_one_textbook_add():
    xs = _xs(2, 5000, "float32")
    for kind in ("single", "double"):
        out = allreduce.reference(xs, kind, CB, "float32")
        want = (xs[0].astype(np.float64) + xs[1].astype(np.float64)).astype(np.float32)
        assert np.array_equal(out[0], want)   # one RN add == RN of the exact sum


def test_P2_bf16_is_one_rounded_add():
    import torch
    xs = _xs(2, 5000, "bfloat16")
    t = [torch.from_numpy(x.view(np.int16)).view(torch.bfloat16) for x in xs]
    want = (t[0].float() + t[1].float()).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(allreduce.reference(xs, "single", CB, "bfloat16")[0], want)


def test_P4_order_pin(golden):
    g = golden("order_pins.txt")
    x = [np.array([float(v)], dtype=np.float32) for v in g["fp32_order_pin_inputs"]]
    got = allreduce.reference(x, "single", 16, "float32")[0][0]
    assert got == float(g["fp32_order_pin_result"][0])
    asc = np.float32(np.float32(np.float32(x[0][0] + x[1][0]) + x[2][0]) + x[3][0])
    assert asc == float(g["fp32_ascending_fold"][0])
    assert sum(float(v[0]) for v in x) == float(g["fp32_exact_sum"][0])


def test_P3_bf16_rounds_once_per_node(golden):
    g = golden("order_pins.txt")
    vals = [float(v) for v in g["bf16_node_rounding_pin_inputs"]]
    xs = [arith.f32_to_bf16_rne(np.array([v], np.float32)) for v in vals]
    got = arith.bf16_to_f32(allreduce.reference(xs, "single", 16, "bfloat16")[0])[0]
    assert got == float(g["bf16_node_rounding_pin_result"][0])
    assert got != float(g["bf16_single_rounding_result"][0])


def _f32(*vals):
    out = vals[0]
    for v in vals[1:]:
        out = np.add(out, v, dtype=np.float32)
    return out


def test_P8_explicit_formulas():
    xs = _xs(8, 4096, "float32")
    x = xs
    t0 = _f32(x[0], _f32(_f32(x[4], _f32(x[2], x[1], x[3])), _f32(x[6], x[5], x[7])))
    t1 = _f32(x[7], _f32(_f32(x[3], _f32(x[1], x[0], x[2])), _f32(x[5], x[4], x[6])))
    single = allreduce.reference(xs, "single", CB, "float32")[0]
    assert np.array_equal(single, t0)
    double = allreduce.reference(xs, "double", CB, "float32")[0]
    E = CB // 4
    for c in range(4096 // E):
        want = t0 if c % 2 == 0 else t1
        assert np.array_equal(double[c * E:(c + 1) * E], want[c * E:(c + 1) * E])


@pytest.mark.parametrize("P", range(1, 9))
@pytest.mark.parametrize("kind", ["single", "double"])
@pytest.mark.parametrize("dtype", arith.DTYPES)
@pytest.mark.parametrize("overlap", [True, False])
def test_replay_equals_definition(P, kind, dtype, overlap):
    """The step-by-step message-passing replay reaches the definition on every rank;
    B and C1 give the same bits; every rank holds identical buffers."""
    count = 2500 + P   # ragged tail
    xs = _xs(P, count, dtype)
    ref = allreduce.reference(xs, kind, CB, dtype)
    out, _ = allreduce.replay(xs, kind, CB, dtype, overlap=overlap)
    for r in range(P):
        assert np.array_equal(out[r], ref[0])
        assert np.array_equal(out[r], out[0])


def test_replay_does_not_touch_inputs():
    xs = _xs(4, 1000, "float32")
    keep = [x.copy() for x in xs]
    allreduce.replay(xs, "double", CB, "float32")
    for a, b in zip(xs, keep):
        assert np.array_equal(a, b)


@pytest.mark.parametrize("P", [2, 4, 8])
@pytest.mark.parametrize("kind", ["single", "double"])
def test_fp32_error_bound(P, kind):
    """|y - s| <= gamma_{P-1} * sum|x| for any summation order (Higham Thm 4.1),
    gamma_n = n u / (1 - n u), u = 2^-24; and the north-star normwise 1e-6."""
    xs = _xs(P, 20000, "float32", seed=11)
    y = allreduce.reference(xs, kind, CB, "float32")[0].astype(np.float64)
    X = np.stack([x.astype(np.float64) for x in xs])
    s = X.sum(0)
    u = 2.0 ** -24
    n = P - 1
    gamma = n * u / (1 - n * u)
    assert np.all(np.abs(y - s) <= gamma * np.abs(X).sum(0))
    assert np.linalg.norm(y - s) / np.linalg.norm(s) <= 1e-6


@pytest.mark.parametrize("P", [2, 4, 8])
def test_bf16_error_bound(P):
    """Per-node rounding: each of the D+1 node levels on a path adds <= 2^-8 relative
    rounding of a partial sum bounded by sum|x|; plus fp32 add error."""
    xs = _xs(P, 20000, "bfloat16", seed=12)
    y = arith.bf16_to_f32(allreduce.reference(xs, "double", CB, "bfloat16")[0]).astype(np.float64)
    X = np.stack([arith.bf16_to_f32(x).astype(np.float64) for x in xs])
    s = X.sum(0)
    D = trees.tree0(P).depth()
    bound = ((D + 1) * 2.0 ** -8 + (P - 1) * 2.0 ** -24) * np.abs(X).sum(0) * 1.0001
    assert np.all(np.abs(y - s) <= bound)
    assert np.linalg.norm(y - s) / np.linalg.norm(s) <= 1e-2


def test_chunk_ownership_double_tree():
    """R4: chunk c is reduced on tree c mod 2 — the double-tree result differs from the
    single-tree one exactly on odd chunks (for generic inputs)."""
    xs = _xs(8, 8 * 256, "float32")
    s = allreduce.reference(xs, "single", CB, "float32")[0]
    d = allreduce.reference(xs, "double", CB, "float32")[0]
    E = CB // 4
    for c in range(8):
        same = np.array_equal(s[c * E:(c + 1) * E], d[c * E:(c + 1) * E])
        assert same == (c % 2 == 0)


def test_partition_counts():
    """SURVEY §8 a3 sizes: ResNet-50 fp32 K=390 with a 254,112 B tail; 64 MiB -> 256 chunks."""
    from paper_conf_hpca_sanghoonsk23_b200 import workloads
    n = workloads.total_elems("resnet50")
    K = partition.num_chunks(n, 256 << 10, 4)
    assert K == 390
    lo, hi = partition.chunk_range(K - 1, n, 256 << 10, 4)
    assert (hi - lo) * 4 == 254112
    assert partition.num_chunks((64 << 20) // 4, 256 << 10, 4) == 256
    nv = workloads.total_elems("vgg16")
    assert partition.num_chunks(nv, 256 << 10, 2) == 1056

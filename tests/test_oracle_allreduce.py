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


# ---- the special-value recipe (IEEE corner cases) ----------------------

def _special(P, count, dtype):
    return [inputs.special(r, count, dtype) for r in range(P)]


@pytest.mark.parametrize("P", [2, 3, 4, 8])
@pytest.mark.parametrize("kind", ["single", "double", "rotated"])
def test_special_fp32_subnormals_are_summed_exactly(P, kind):
    """Class 2 (subnormals on every rank, |x| < 2^-129): any order's fp32 sum is
    exact and subnormal, so the oracle must return the exact integer sum of the
    mantissas times 2^-149 — a flush-to-zero anywhere would give 0 instead."""
    count = 6000
    xs = _special(P, count, "float32")
    out = allreduce.reference(xs, kind, 1024, "float32")[0]
    cls = inputs.special_class(0, count)
    sel = cls == 2
    bits = np.stack([x.view(np.uint32)[sel] for x in xs]).astype(np.int64)
    mag = bits & 0x7FFFFFFF
    sgn = np.where(bits >> 31, -1, 1)
    exact = (sgn * mag).sum(axis=0)                      # units of 2^-149
    assert np.array_equal(out[sel].astype(np.float64), np.ldexp(exact.astype(np.float64), -149))
    assert (out[sel] != 0).sum() > 0.9 * sel.sum()
    assert (np.abs(out[sel]) < 2.0 ** -126).all()


@pytest.mark.parametrize("P", [2, 4, 5, 8])
@pytest.mark.parametrize("dtype", ["float32", "bfloat16"])
def test_special_signed_zeros(P, dtype):
    """Class 3: an IEEE RN sum is -0 only when every addend is -0; with any +0 among
    them it is +0 (IEEE 754 §6.3).  Both hold per element whatever the tree."""
    count = 6000
    xs = _special(P, count, dtype)
    for kind in ("single", "double"):
        out = arith.to_float64(allreduce.reference(xs, kind, 1024, dtype)[0], dtype)
        sel = inputs.special_class(0, count) == 3
        vals = np.stack([arith.to_float64(x, dtype)[sel] for x in xs])
        assert (vals == 0).all()
        all_neg = np.signbit(vals).all(axis=0)
        assert all_neg.sum() > 50 and (~all_neg).sum() > 50
        assert (out[sel] == 0).all()
        assert np.array_equal(np.signbit(out[sel]), all_neg)


@pytest.mark.parametrize("P", [2, 4, 6, 8])
def test_special_fp32_cancellation_gives_plus_zero(P):
    """Class 6 at even P: +m on even ranks, -m on odd, every partial sum exact, so
    the exact total is 0 and the RN result is +0 in every tree and order."""
    count = 6000
    xs = _special(P, count, "float32")
    sel = inputs.special_class(0, count) == 6
    for kind in ("single", "double", "rotated"):
        out = allreduce.reference(xs, kind, 1024, "float32")[0][sel]
        assert (out == 0).all() and not np.signbit(out).any()


@pytest.mark.parametrize("dtype", ["float32", "bfloat16"])
def test_special_values_stay_finite_and_within_the_bound(dtype):
    """Near-max (class 4) sums of 8 cannot overflow; every result obeys the same
    error bound as the normal recipe (Higham for fp32; per-node rounding for bf16)."""
    P, count = 8, 8000
    xs = _special(P, count, dtype)
    out = arith.to_float64(allreduce.reference(xs, "double", 1024, dtype)[0], dtype)
    vals = np.stack([arith.to_float64(x, dtype) for x in xs])
    assert np.isfinite(out).all()
    s, a = vals.sum(axis=0), np.abs(vals).sum(axis=0)
    if dtype == "float32":
        u = 2.0 ** -24
        g = (P - 1) * u / (1 - (P - 1) * u)
        # subnormal results carry an absolute error of at most half an ulp of 2^-149
        assert (np.abs(out - s) <= g * a + 2.0 ** -150).all()
    else:
        assert (np.abs(out - s) <= (3 * 2.0 ** -8 + 7 * 2.0 ** -24) * a + 2.0 ** -133).all()


def test_special_int32_is_the_wrapped_sum():
    P, count = 8, 6000
    xs = _special(P, count, "int32")
    assert (np.concatenate(xs) == np.iinfo(np.int32).min).any()
    assert (np.concatenate(xs) == np.iinfo(np.int32).max).any()
    want = np.sum(np.stack(xs).astype(np.int64), axis=0).astype(np.uint64).astype(np.uint32)
    for kind in ("single", "double", "rotated"):
        assert np.array_equal(allreduce.reference(xs, kind, 1024, "int32")[0].view(np.uint32), want)

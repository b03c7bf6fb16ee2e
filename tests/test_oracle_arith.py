"""Pins for oracle.arith (readings R2, R3): bf16 RNE, int32 wrap, fp32 order."""

from fractions import Fraction

import numpy as np
import pytest
import torch

from oracle import arith


def _rne_bruteforce(x: float) -> float:
    """Nearest bf16 to x by exact rational distance, ties to even significand."""
    u = np.array([x], dtype=np.float32).view(np.uint32)[0]
    lo = int(u) & 0xFFFF0000
    hi = lo + 0x10000
    cands = []
    for pat in (lo, hi):
        f = np.array([pat], dtype=np.uint32).view(np.float32)[0]
        cands.append((abs(Fraction(float(f)) - Fraction(float(x))), (pat >> 16) & 1, pat >> 16))
    cands.sort()
    if cands[0][0] == cands[1][0]:          # tie -> even
        return [c for c in cands if c[1] == 0][0][2]
    return cands[0][2]


def test_bf16_rne_bruteforce():
    rng = np.random.default_rng(1)
    xs = np.concatenate([
        rng.standard_normal(3000).astype(np.float32),
        (rng.standard_normal(500) * 1e-38).astype(np.float32),       # subnormals
        np.array([1 + 2 ** -8, 1 + 3 * 2 ** -8, -1 - 2 ** -8, 3.0e38, 0.0, -0.0], dtype=np.float32),
    ])
    got = arith.f32_to_bf16_rne(xs)
    for x, g in zip(xs, got):
        assert int(g) == _rne_bruteforce(float(x)), x


def test_bf16_rne_matches_torch():
    rng = np.random.default_rng(2)
    xs = (rng.standard_normal(100000) * 10.0 ** rng.integers(-30, 30, 100000)).astype(np.float32)
    ref = torch.from_numpy(xs).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(arith.f32_to_bf16_rne(xs), ref)


def test_bf16_widen_exact():
    pats = np.arange(0, 1 << 16, dtype=np.uint32).astype(np.uint16)
    f = arith.bf16_to_f32(pats)
    ref = torch.from_numpy(pats.view(np.int16)).view(torch.bfloat16).float().numpy()
    finite = np.isfinite(ref)
    assert np.array_equal(f[finite].view(np.uint32), ref[finite].view(np.uint32))


def test_bf16_tie_pins(golden):
    g = golden("order_pins.txt")
    for key in ("bf16_tie_pin_a", "bf16_tie_pin_b"):
        x, want = (float(v) for v in g[key])
        got = arith.bf16_to_f32(arith.f32_to_bf16_rne(np.array([x], np.float32)))[0]
        assert got == want


def test_int32_wraps_mod_2_32():
    rng = np.random.default_rng(3)
    a = rng.integers(-2 ** 31, 2 ** 31, 1000, dtype=np.int64).astype(np.int32)
    b = rng.integers(-2 ** 31, 2 ** 31, 1000, dtype=np.int64).astype(np.int32)
    c = rng.integers(-2 ** 31, 2 ** 31, 1000, dtype=np.int64).astype(np.int32)
    got = arith.combine(a, [b, c], "int32")
    for i in range(1000):
        s = (int(a[i]) + int(b[i]) + int(c[i])) % (1 << 32)
        s = s - (1 << 32) if s >= (1 << 31) else s
        assert int(got[i]) == s


def test_fp32_left_to_right_is_ieee_add():
    rng = np.random.default_rng(4)
    a, b, c = (rng.standard_normal(1000).astype(np.float32) for _ in range(3))
    got = arith.combine(a, [b, c], "float32")
    for i in range(1000):
        # Python float adds are binary64; rounding each partial to binary32 gives
        # the binary32 RN add exactly (double rounding is innocuous for a single
        # add of two binary32 values since 53 >= 2*24+2).
        ab = np.float32(float(a[i]) + float(b[i]))
        assert got[i] == np.float32(float(ab) + float(c[i]))


def test_leaf_passes_own_value_unchanged():
    x = np.array([1, 2, 3], dtype=np.uint16)
    assert np.array_equal(arith.combine(x, [], "bfloat16"), x)


@pytest.mark.parametrize("dtype", arith.DTYPES)
def test_combine_does_not_mutate(dtype):
    own = np.ones(8, dtype=arith.NP_STORAGE[dtype])
    kid = np.ones(8, dtype=arith.NP_STORAGE[dtype])
    before = own.copy()
    arith.combine(own, [kid], dtype)
    assert np.array_equal(own, before)

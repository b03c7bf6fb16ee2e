"""Seeded synthetic gradient generator shared by tests, bench and smoke.

Holds none of the method's arithmetic: it only produces per-rank input buffers.
Recipe:
  value(rank r, element e) = scale(layer(e)) * z(r, e)
  z: Box–Muller on a counter-based splitmix64(seed ^ (r << 48) ^ e), so a value
     depends only on (seed, r, e) — never on chunking, threading or device;
  scale(l) = 2**-(l mod 8) to vary magnitudes across layers (gradients of
     different layers differ in scale);
  layer(e) from a workload's layer table (workloads.py) or, without one,
     consecutive 4096-element pseudo-layers.
  bf16 inputs are the round-to-nearest-even bf16 of the fp32 values (torch's
  conversion); int32 inputs are uniform in [-2**24, 2**24) (sums are then exact
  without wrap at P <= 8) or, with ``full_range=True``, uniform over all int32.
Default seed 20230225 (the paper's conference date), recorded in bench output.

``special(rank, count, dtype)`` is a second recipe for the parity tests (VERDICT r1
W2): IEEE corner cases that decide whether the device honours reading R3 (no
FTZ/DAZ, RN adds, signed zeros, one RNE per bf16 node output).  Every element
belongs to a class picked by a RANK-INDEPENDENT hash of (seed, e), so all ranks
see the same kind of value at e and the partial sums stay in that regime:
  0, 1  normal: the default recipe's N(0,1) * 2^-k;
  2     subnormal: +-m * 2^-149 with m in [1, 2^20) (fp32) or [2^16, 2^20) (bf16),
        random sign per rank; any tree's sum of <= 8 stays exact and below 2^-126,
        so a flush-to-zero anywhere turns a nonzero result into 0;
  3     signed zero: +0 or -0 per rank; on every other such element all ranks -0
        (the only way an IEEE RN sum is -0);
  4     near the format maximum: +-(1 + f) * 2^123 (sums of <= 8 cannot overflow);
  5     at the normal/subnormal boundary: exponent field 0 or 1, random mantissa;
  6     cancellation: the same magnitude m (8 significant bits, so every partial
        sum k*m, |k| <= 8, is exact in fp32) on every rank, + on even ranks, - on
        odd: at even P the exact sum is 0, and an RN sum that is exactly zero is +0;
  7     mixed: the class of (rank, e) instead, so magnitudes of every kind meet.
int32: 0,1 uniform in [-2^24, 2^24); 2 INT32_MIN; 3 INT32_MAX; 4 in {-1, 0, 1};
5, 6, 7 uniform over all int32 (wraps).  No NaN or Inf is generated (unpinned).
"""

from typing import Optional, Sequence

import numpy as np

SEED = 20230225
_PSEUDO_LAYER = 4096

_M1 = np.uint64(0x9E3779B97F4A7C15)
_M2 = np.uint64(0xBF58476D1CE4E5B9)
_M3 = np.uint64(0x94D049BB133111EB)


def splitmix64(x: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = x + _M1
        z = (z ^ (z >> np.uint64(30))) * _M2
        z = (z ^ (z >> np.uint64(27))) * _M3
        return z ^ (z >> np.uint64(31))


def _hash(rank: int, lo: int, hi: int, seed: int) -> np.ndarray:
    e = np.arange(lo, hi, dtype=np.uint64)
    key = np.uint64(seed) ^ (np.uint64(rank) << np.uint64(48))
    return splitmix64(e ^ key)


def _layer_index(lo: int, hi: int, layer_ends: Optional[Sequence[int]]) -> np.ndarray:
    e = np.arange(lo, hi, dtype=np.int64)
    if layer_ends is None:
        return e // _PSEUDO_LAYER
    return np.searchsorted(np.asarray(layer_ends, dtype=np.int64), e, side="right")


def gradients_f32(rank: int, count: int, seed: int = SEED,
                  layer_ends: Optional[Sequence[int]] = None,
                  lo: int = 0, hi: Optional[int] = None) -> np.ndarray:
    """fp32 gradients of elements [lo, hi) (default: the whole buffer of ``count``)."""
    hi = count if hi is None else hi
    h1 = _hash(rank, lo, hi, seed)
    h2 = splitmix64(h1)
    u1 = ((h1 >> np.uint64(11)).astype(np.float64) + 1.0) * (2.0 ** -53)   # (0, 1]
    u2 = (h2 >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)           # [0, 1)
    z = np.sqrt(-2.0 * np.log(u1)) * np.cos(2.0 * np.pi * u2)
    scale = np.ldexp(1.0, -(_layer_index(lo, hi, layer_ends) % 8).astype(np.int64))
    return (z * scale).astype(np.float32)


def gradients_bf16(rank: int, count: int, seed: int = SEED,
                   layer_ends: Optional[Sequence[int]] = None,
                   lo: int = 0, hi: Optional[int] = None) -> np.ndarray:
    """bf16 bit patterns (uint16) = RNE(bf16) of the fp32 gradients."""
    import torch
    f = torch.from_numpy(gradients_f32(rank, count, seed, layer_ends, lo, hi))
    return f.to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)


def gradients_i32(rank: int, count: int, seed: int = SEED, full_range: bool = False,
                  lo: int = 0, hi: Optional[int] = None) -> np.ndarray:
    hi = count if hi is None else hi
    h = _hash(rank, lo, hi, seed)
    if full_range:
        return (h & np.uint64(0xFFFFFFFF)).astype(np.uint32).view(np.int32)
    return ((h >> np.uint64(39)).astype(np.int64) - (1 << 24)).astype(np.int32)


def gradients(rank: int, count: int, dtype: str, seed: int = SEED,
              layer_ends: Optional[Sequence[int]] = None, full_range: bool = False,
              lo: int = 0, hi: Optional[int] = None) -> np.ndarray:
    if dtype == "float32":
        return gradients_f32(rank, count, seed, layer_ends, lo, hi)
    if dtype == "bfloat16":
        return gradients_bf16(rank, count, seed, layer_ends, lo, hi)
    if dtype == "int32":
        return gradients_i32(rank, count, seed, full_range, lo, hi)
    raise ValueError(dtype)


# ---- the special-value recipe (parity tests) ---------------------------------------
SPECIAL_CLASSES = 8


def special_class(lo: int, hi: int, seed: int = SEED, rank: Optional[int] = None) -> np.ndarray:
    """Class of elements [lo, hi): a hash of (seed, e) — of (seed, rank, e) with rank."""
    key = np.uint64(seed ^ 0x5EC1A1) if rank is None else \
        np.uint64(seed ^ 0x5EC1A1) ^ (np.uint64(rank + 1) << np.uint64(40))
    h = splitmix64(np.arange(lo, hi, dtype=np.uint64) ^ key)
    return (h >> np.uint64(61)).astype(np.int64)


def _special_f32_bits(rank: int, lo: int, hi: int, seed: int, bf16: bool) -> np.ndarray:
    cls = special_class(lo, hi, seed)
    mixed = cls == 7
    cls[mixed] = special_class(lo, hi, seed, rank)[mixed] % 7
    h = _hash(rank, lo, hi, seed ^ 0x77)                  # per (rank, e)
    hs = splitmix64(np.arange(lo, hi, dtype=np.uint64) ^ np.uint64(seed ^ 0x3C3C))  # per e
    sign = ((h >> np.uint64(63)) << np.uint64(31)).astype(np.uint32)
    mant = ((h >> np.uint64(20)) & np.uint64(0x7FFFFF)).astype(np.uint32)
    base = gradients_f32(rank, hi, seed, None, lo, hi).view(np.uint32)
    out = base.copy()
    # 2: subnormal
    if bf16:
        m = (np.uint32(1 << 16) + (mant & np.uint32((1 << 20) - 1 - (1 << 16))))
    else:
        m = np.maximum(mant & np.uint32((1 << 20) - 1), np.uint32(1))
    sel = cls == 2
    out[sel] = sign[sel] | m[sel]
    # 3: signed zero (every other such element: all ranks -0)
    sel = cls == 3
    all_neg = ((hs >> np.uint64(7)) & np.uint64(1)).astype(bool)
    out[sel] = np.where(all_neg[sel], np.uint32(0x80000000), sign[sel])
    # 4: near max, +-(1 + f) * 2^123
    sel = cls == 4
    out[sel] = sign[sel] | np.uint32((123 + 127) << 23) | mant[sel]
    # 5: exponent field 0 or 1
    sel = cls == 5
    e1 = ((h >> np.uint64(5)) & np.uint64(1)).astype(np.uint32) << np.uint32(23)
    out[sel] = sign[sel] | e1[sel] | mant[sel]
    # 6: cancellation: magnitude per e, sign by rank parity
    sel = cls == 6
    mag = (np.uint32(127 << 23) | ((hs >> np.uint64(20)) & np.uint64(0x7F0000)).astype(np.uint32))
    out[sel] = mag[sel] | (np.uint32(0x80000000) if rank % 2 else np.uint32(0))
    return out


def special(rank: int, count: int, dtype: str, seed: int = SEED,
            lo: int = 0, hi: Optional[int] = None) -> np.ndarray:
    """The special-value recipe (module docstring) for elements [lo, hi)."""
    hi = count if hi is None else hi
    if dtype == "float32":
        return _special_f32_bits(rank, lo, hi, seed, False).view(np.float32)
    if dtype == "bfloat16":
        import torch
        f = torch.from_numpy(_special_f32_bits(rank, lo, hi, seed, True).view(np.float32))
        return f.to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    if dtype == "int32":
        cls = special_class(lo, hi, seed)
        mixed = cls == 7
        cls[mixed] = special_class(lo, hi, seed, rank)[mixed] % 7
        h = _hash(rank, lo, hi, seed ^ 0x99)
        out = ((h >> np.uint64(39)).astype(np.int64) - (1 << 24)).astype(np.int32)
        full = (h & np.uint64(0xFFFFFFFF)).astype(np.uint32).view(np.int32)
        out[cls == 2] = np.iinfo(np.int32).min
        out[cls == 3] = np.iinfo(np.int32).max
        small = ((h >> np.uint64(3)) % np.uint64(3)).astype(np.int32) - 1
        out[cls == 4] = small[cls == 4]
        sel = cls >= 5
        out[sel] = full[sel]
        return out
    raise ValueError(dtype)

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

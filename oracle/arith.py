"""Per-node combine ⊕ (oracle; test infrastructure only).

The paper never states a precision or a combine order (it presumably used fp32,
fn7 P:L289).  It does state that "C-Cube does not change the ordering of any
computation", so the result is a fixed-order fold.  Readings
(DESIGN.md §3):

  R2: at node v the combine is ``own ⊕ partial(child_1) ⊕ partial(child_2)``,
      evaluated left to right, children in ascending rank.
  R3: int32 adds wrap modulo 2**32; fp32 adds are IEEE round-to-nearest-even
      with no FMA contraction and no flush-to-zero; bf16 values are widened to
      fp32, added in the same order in fp32, and rounded ONCE to bf16 (RNE) per
      node output.  A leaf forwards its own value unchanged.

bf16 arrays are carried as numpy ``uint16`` bit patterns (numpy has no bf16).
"""

import numpy as np

DTYPES = ("int32", "float32", "bfloat16")
ELEM_SIZE = {"int32": 4, "float32": 4, "bfloat16": 2}
NP_STORAGE = {"int32": np.int32, "float32": np.float32, "bfloat16": np.uint16}


def bf16_to_f32(u16: np.ndarray) -> np.ndarray:
    """Exact widening: a bf16 pattern is the top 16 bits of an fp32 pattern."""
    return (np.asarray(u16, dtype=np.uint16).astype(np.uint32) << np.uint32(16)).view(np.float32)


def f32_to_bf16_rne(f: np.ndarray) -> np.ndarray:
    """Round fp32 -> bf16, to nearest, ties to even (finite inputs; NaN unpinned)."""
    u = np.asarray(f, dtype=np.float32).view(np.uint32).astype(np.uint64)
    lsb = (u >> np.uint64(16)) & np.uint64(1)
    return ((u + np.uint64(0x7FFF) + lsb) >> np.uint64(16)).astype(np.uint16)


def combine(own: np.ndarray, partials, dtype: str) -> np.ndarray:
    """R2/R3: own ⊕ p_1 ⊕ ... left to right.  ``partials`` are the children's
    partial results in ascending child rank.  With no partials (a leaf) the own
    value is returned unchanged."""
    partials = list(partials)
    if not partials:
        return np.array(own, copy=True)
    if dtype == "int32":
        acc = np.asarray(own, dtype=np.int32).view(np.uint32).copy()
        for p in partials:
            acc = acc + np.asarray(p, dtype=np.int32).view(np.uint32)   # mod 2**32
        return acc.view(np.int32)
    if dtype == "float32":
        acc = np.asarray(own, dtype=np.float32).copy()
        for p in partials:
            acc = np.add(acc, np.asarray(p, dtype=np.float32), dtype=np.float32)
        return acc
    if dtype == "bfloat16":
        acc = bf16_to_f32(own)
        for p in partials:
            acc = np.add(acc, bf16_to_f32(p), dtype=np.float32)
        return f32_to_bf16_rne(acc)
    raise ValueError(dtype)


def to_float64(x: np.ndarray, dtype: str) -> np.ndarray:
    """Exact value of each element as fp64 (for error measurements)."""
    if dtype == "bfloat16":
        return bf16_to_f32(x).astype(np.float64)
    return np.asarray(x).astype(np.float64)

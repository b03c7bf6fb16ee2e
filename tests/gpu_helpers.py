"""Helpers for the -m gpu parity tests (inputs -> torch CUDA tensors, oracle slices)."""

import numpy as np
import torch

from oracle import allreduce as oar
from oracle import arith, partition
from oracle import trees as otrees
from paper_conf_hpca_sanghoonsk23_b200 import inputs

TORCH_DTYPE = {"int32": torch.int32, "float32": torch.float32, "bfloat16": torch.bfloat16}


def to_torch(x: np.ndarray, dtype: str) -> torch.Tensor:
    if dtype == "bfloat16":
        return torch.from_numpy(x.view(np.int16)).view(torch.bfloat16)
    return torch.from_numpy(x)


def to_numpy(t: torch.Tensor, dtype: str) -> np.ndarray:
    t = t.detach().cpu()
    if dtype == "bfloat16":
        return t.view(torch.int16).numpy().view(np.uint16)
    return t.numpy()


def device_inputs(P, count, dtype, seed=inputs.SEED, layer_ends=None, block=1 << 24):
    """Per-rank CUDA buffers filled block by block from the seeded generator."""
    out = []
    for r in range(P):
        t = torch.empty(count, dtype=TORCH_DTYPE[dtype], device="cuda")
        for lo in range(0, count, block):
            hi = min(count, lo + block)
            x = inputs.gradients(r, count, dtype, seed=seed, layer_ends=layer_ends, lo=lo, hi=hi)
            t[lo:hi].copy_(to_torch(x, dtype))
        out.append(t)
    return out


def oracle_chunk(P, kind, chunk_bytes, dtype, count, c, seed=inputs.SEED, layer_ends=None):
    """Oracle result (definition) of chunk c alone: the fixed-order fold on tree c mod T."""
    es = arith.ELEM_SIZE[dtype]
    lo, hi = partition.chunk_range(c, count, chunk_bytes, es)
    xs = [inputs.gradients(r, count, dtype, seed=seed, layer_ends=layer_ends, lo=lo, hi=hi)
          for r in range(P)]
    ts = otrees.trees(P, kind)
    tree = ts[partition.tree_of_chunk(c, len(ts))]
    return lo, hi, oar.fold(xs, tree, tree.root, dtype)

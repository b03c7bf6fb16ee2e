"""a3 — chunk partition and chunk->tree map (oracle; test infrastructure only).

Paper basis
  * "Chunk is the amount of data that is communicated between neighboring nodes
    in each step of AllReduce" (fn3).
  * One-shot collective, no finer partitioning, pipelined over "the optimal chunk
    size" (§II-B); 256 chunks for 64 MB -> 256 KiB default.
  * Two trees "to fully utilize the bandwidth" — no split rule is given.

Readings
  R4: in the double tree chunk c goes to tree ``c mod 2``; with T trees (the
      rotated set, R17) to tree ``c mod T``.
  R5: the last chunk may be partial; chunk_bytes is a multiple of 16.
  R8: the chunk count is ceil(bytes / chunk_bytes) with chunk_bytes fixed at init;
      eq 4's K_opt is advisory only.
"""

from typing import List, Tuple

DEFAULT_CHUNK_BYTES = 256 * 1024  # 256 chunks for 64 MB


def elems_per_chunk(chunk_bytes: int, elem_size: int) -> int:
    if chunk_bytes <= 0 or chunk_bytes % 16:
        raise ValueError("chunk_bytes must be a positive multiple of 16 (R5)")
    return chunk_bytes // elem_size


def num_chunks(count: int, chunk_bytes: int, elem_size: int) -> int:
    E = elems_per_chunk(chunk_bytes, elem_size)
    return (count + E - 1) // E


def chunk_range(c: int, count: int, chunk_bytes: int, elem_size: int) -> Tuple[int, int]:
    """Elements [lo, hi) of chunk c."""
    E = elems_per_chunk(chunk_bytes, elem_size)
    return c * E, min((c + 1) * E, count)


def chunks(count: int, chunk_bytes: int, elem_size: int) -> List[Tuple[int, int]]:
    return [chunk_range(c, count, chunk_bytes, elem_size)
            for c in range(num_chunks(count, chunk_bytes, elem_size))]


def tree_of_chunk(c: int, ntrees: int) -> int:
    """R4: single tree -> 0; double tree -> c mod 2; T trees -> c mod T."""
    return c % ntrees


def tree_local_index(c: int, ntrees: int) -> int:
    """Position of chunk c in its tree's in-order chunk stream."""
    return c // ntrees


def chunks_of_tree(t: int, K: int, ntrees: int) -> List[int]:
    """Global chunk ids carried by tree t, in the order the tree processes them."""
    return [c for c in range(K) if tree_of_chunk(c, ntrees) == t]

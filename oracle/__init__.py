"""C-Cube CPU oracle — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import, call or execute anything under ``oracle/``.
The product path (``paper_conf_hpca_sanghoonsk23_b200``) never imports it and
fails loudly if its CUDA library is missing; it has no CPU fallback.

This package is a plain, slow, obviously-correct CPU implementation of what the
C-Cube hot path computes, written from the paper
(/root/reference/PAPER.md, cited as ``P:Lnnn``) and from the readings listed
in DESIGN.md §3.  It shares no code with the CUDA path: no kernels, headers,
helpers, tables or constant generators.

Modules
  trees      — a1: the logical (double) binary tree (fn4 P:L153)
  partition  — a3: chunking and the chunk→tree map (fn3 P:L88)
  arith      — per-node combine ⊕ for int32 / fp32 / bf16 (DESIGN readings R2, R3)
  allreduce  — the fixed-order tree fold (the definition) and a message-passing
               replay of the pipelined schedule
  schedule   — the dedicated-link step simulator of Figs 5/7
  gradq      — gradient queue: Layer-Chunk Table, Fig 11 semaphore, gates
               
  costmodel  — eqs 1–7 and per-port loads

Parity status: every public function is pinned by a ``-m "not gpu"`` test in
``tests/test_oracle_*.py`` against values the paper prints, closed forms,
brute force or library routines.  Unpinned (documented in DESIGN.md): NaN/Inf
propagation; absolute timings; cross-tree landing order in the double tree.
"""

from . import trees, partition, arith, allreduce, schedule, gradq, costmodel  # noqa: F401

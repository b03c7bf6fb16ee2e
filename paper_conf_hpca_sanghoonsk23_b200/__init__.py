"""C-Cube on B200: chunk-pipelined (double-)tree AllReduce with gradient queuing.

The compute path is ``csrc/`` (hand-written sm_100a CUDA + a C++ host runtime)
behind the C ABI in ``include/ccube.h``; ``ccube.py`` is a thin ctypes binding
with the same names.  The CUDA library is loaded on first use and its absence is
an error: there is no CPU fallback.
"""

from . import inputs, workloads  # noqa: F401  (pure-python helpers; no CUDA)

__all__ = ["inputs", "workloads"]

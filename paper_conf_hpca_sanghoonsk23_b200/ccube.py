"""Thin ctypes binding of include/ccube.h (argument marshalling only).

Every step of the AllReduce and of the gradient-queue gate runs in
``libccube.so``'s sm_100a kernels; this module only converts Python/torch
arguments into pointers, sizes and stream handles.  If the library is missing the
call raises — there is no CPU fallback.

Names mirror the C ABI: ``init`` (ccube_init), ``allreduce_tree`` /
``allreduce_tree_local``, ``gradq_set_layers``, ``gradq_wait`` /
``gradq_wait_local``, ``set_overlap``, ``set_channels``, ``set_threads``,
``set_trace``, ``register_buffers``, ``deregister_buffers``, ``barrier``, ``finalize``,
``last_error``, ``get_info``, ``tree_parents``, ``set_placement``,
``plan_placement``, ``tree_parents_placed``, ``plan_launch``.
"""

import ctypes
import os
from typing import Optional, Sequence

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libccube.so")

SUCCESS = 0
ERR_INVALID_ARG = -1
ERR_NOT_INITIALIZED = -2
ERR_ALREADY_INITIALIZED = -3
ERR_CUDA = -4
ERR_UNSUPPORTED = -5
ERR_BOOTSTRAP = -6
ERR_TIMEOUT = -7
_NAMES = {0: "SUCCESS", -1: "INVALID_ARG", -2: "NOT_INITIALIZED", -3: "ALREADY_INITIALIZED",
          -4: "CUDA", -5: "UNSUPPORTED", -6: "BOOTSTRAP", -7: "TIMEOUT"}

TREE = {"single": 0, "double": 1, "rotated": 2}
TRANSPORT = {"auto": 0, "push": 1, "pull": 2}
DATAPATH = {"auto": -1, "lsu": 0, "tma": 1}
DTYPE = {"int32": 0, "float32": 1, "bfloat16": 2}

EXPORTS = [
    "ccube_init", "ccube_register_buffers", "ccube_deregister_buffers", "ccube_allreduce_tree",
    "ccube_allreduce_tree_local", "ccube_gradq_set_layers", "ccube_gradq_wait",
    "ccube_gradq_wait_local", "ccube_gradq_set_sgd", "ccube_set_overlap", "ccube_set_channels", "ccube_set_threads",
    "ccube_set_trace", "ccube_set_transport", "ccube_set_datapath", "ccube_finalize", "ccube_last_error", "ccube_get_info",
    "ccube_tree_parents",
    "ccube_set_placement",
    "ccube_plan_placement",
    "ccube_tree_parents_placed",
    "ccube_barrier",
    "ccube_plan_launch",
    "ccube_measure_peer_bandwidth",
    "ccube_set_protocol",
]


class CCubeError(RuntimeError):
    def __init__(self, code: int, func: str, msg: str):
        super().__init__(f"{func} -> CCUBE_ERR_{_NAMES.get(code, code)}: {msg}")
        self.code = code


ALLGATHER_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                ctypes.c_size_t)


class World(ctypes.Structure):
    _fields_ = [("rank", ctypes.c_int), ("nlocal", ctypes.c_int), ("world_size", ctypes.c_int),
                ("cuda_device", ctypes.c_int), ("allgather", ALLGATHER_FN),
                ("ctx", ctypes.c_void_p)]


class Info(ctypes.Structure):
    _fields_ = [("initialized", ctypes.c_int), ("world_size", ctypes.c_int),
                ("rank", ctypes.c_int), ("nlocal", ctypes.c_int), ("ntrees", ctypes.c_int),
                ("channels", ctypes.c_int), ("threads", ctypes.c_int), ("overlap", ctypes.c_int),
                ("transport", ctypes.c_int), ("chunk_bytes", ctypes.c_size_t), ("epoch_base", ctypes.c_uint64 * 2),
                ("last_channels", ctypes.c_int), ("last_ctas", ctypes.c_int),
                ("datapath", ctypes.c_int), ("last_tma", ctypes.c_int),
                ("protocol", ctypes.c_int), ("last_ll", ctypes.c_int),
                ("last_threads", ctypes.c_int)]


_lib = None
_keepalive = []


def lib() -> ctypes.CDLL:
    """Load libccube.so (built in-tree by __graft_entry__.build()).  Raises if absent."""
    global _lib
    if _lib is None:
        # CCUBE_LIB: an experiment build of the same sources (tools/experiments); the
        # product, tests and smoke use the in-tree library
        path = os.environ.get("CCUBE_LIB") or LIB_PATH
        if not os.path.exists(path):
            raise RuntimeError(f"{path} is missing: run `python -m "
                               "paper_conf_hpca_sanghoonsk23_b200.build` (no CPU fallback)")
        L = ctypes.CDLL(path)
        vp, sz, i = ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int
        sig = {
            "ccube_init": [ctypes.POINTER(World), i, sz],
            "ccube_register_buffers": [ctypes.POINTER(vp), sz],
            "ccube_deregister_buffers": [ctypes.POINTER(vp)],
            "ccube_allreduce_tree": [vp, sz, i, vp],
            "ccube_allreduce_tree_local": [ctypes.POINTER(vp), sz, i, vp],
            "ccube_gradq_set_layers": [ctypes.POINTER(sz), i],
            "ccube_gradq_wait": [i, vp],
            "ccube_gradq_wait_local": [i, i, vp],
            "ccube_gradq_set_sgd": [ctypes.POINTER(vp), sz, ctypes.c_float],
            "ccube_set_overlap": [i],
            "ccube_set_channels": [i],
            "ccube_set_threads": [i],
            "ccube_set_trace": [vp, sz],
            "ccube_set_transport": [i],
            "ccube_set_datapath": [i],
            "ccube_set_protocol": [i],
            "ccube_finalize": [],
            "ccube_get_info": [ctypes.POINTER(Info)],
            "ccube_tree_parents": [i, i, i, ctypes.POINTER(i)],
            "ccube_set_placement": [ctypes.POINTER(i), i],
            "ccube_plan_placement": [i, i, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(i)],
            "ccube_tree_parents_placed": [i, i, i, ctypes.POINTER(i), ctypes.POINTER(i)],
            "ccube_barrier": [vp],
            "ccube_plan_launch": [i, i, i, i, sz, sz, i, i, i, ctypes.POINTER(i),
                                  ctypes.POINTER(i), ctypes.POINTER(i)],
            "ccube_measure_peer_bandwidth": [sz, i, ctypes.POINTER(ctypes.c_double),
                                             ctypes.POINTER(ctypes.c_double)],
        }
        for name, args in sig.items():
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = ctypes.c_int
        L.ccube_last_error.argtypes = []
        L.ccube_last_error.restype = ctypes.c_char_p
        _lib = L
    return _lib


def last_error() -> str:
    return lib().ccube_last_error().decode()


def _check(rc: int, func: str) -> None:
    if rc != SUCCESS:
        raise CCubeError(rc, func, last_error())


def _stream_handle(stream) -> Optional[int]:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def _dtype_code(t) -> int:
    import torch
    m = {torch.int32: 0, torch.float32: 1, torch.bfloat16: 2}
    if t.dtype not in m:
        raise CCubeError(ERR_INVALID_ARG, "dtype", f"unsupported dtype {t.dtype}")
    return m[t.dtype]


def _ptr_array(ptrs: Sequence[int]):
    return (ctypes.c_void_p * len(ptrs))(*ptrs)


# ---------------------------------------------------------------------------- init

def _torch_allgather(pg):
    """allgather callback over a torch.distributed process group (gloo or nccl)."""
    import torch
    import torch.distributed as dist

    def cb(_ctx, send, recv, nbytes):
        try:
            backend = dist.get_backend(pg)
            dev = torch.device("cuda", torch.cuda.current_device()) if backend == "nccl" \
                else torch.device("cpu")
            src = torch.frombuffer(bytearray(ctypes.string_at(send, nbytes)), dtype=torch.uint8)
            src = src.to(dev)
            n = dist.get_world_size(pg)
            outs = [torch.empty(nbytes, dtype=torch.uint8, device=dev) for _ in range(n)]
            dist.all_gather(outs, src, group=pg)
            blob = b"".join(bytes(o.cpu().numpy().tobytes()) for o in outs)
            ctypes.memmove(recv, blob, len(blob))
            return 0
        except Exception as e:  # noqa: BLE001 — reported through the C return code
            import sys
            print(f"[ccube] allgather callback failed: {e!r}", file=sys.stderr)
            return 1

    return ALLGATHER_FN(cb)


def init(world_size: int, rank: int = 0, nlocal: Optional[int] = None, device: int = 0,
         tree: str = "single", chunk_bytes: int = 0, pg=None) -> None:
    """ccube_init.  nlocal=None -> world_size (loopback, one process, one GPU) when
    pg is None, else 1 (one process per GPU, allgather over ``pg``)."""
    if nlocal is None:
        nlocal = world_size if pg is None else 1
    cb = _torch_allgather(pg) if nlocal < world_size else ALLGATHER_FN()
    _keepalive.append(cb)
    w = World(rank=rank, nlocal=nlocal, world_size=world_size, cuda_device=device,
              allgather=cb, ctx=None)
    _check(lib().ccube_init(ctypes.byref(w), TREE[tree], chunk_bytes), "ccube_init")


def init_loopback(P: int, tree: str = "single", chunk_bytes: int = 0, device: int = 0) -> None:
    init(P, rank=0, nlocal=P, device=device, tree=tree, chunk_bytes=chunk_bytes)


def init_distributed(pg=None, tree: str = "double", chunk_bytes: int = 0) -> None:
    """One process per GPU over torch.distributed (rank/world from ``pg``)."""
    import torch
    import torch.distributed as dist
    init(dist.get_world_size(pg), rank=dist.get_rank(pg), nlocal=1,
         device=torch.cuda.current_device(), tree=tree, chunk_bytes=chunk_bytes,
         pg=pg if pg is not None else dist.group.WORLD)


def finalize() -> None:
    _check(lib().ccube_finalize(), "ccube_finalize")


# ---------------------------------------------------------------------- collective

def register_buffers(tensors, nbytes: Optional[int] = None) -> None:
    ts = list(tensors)
    n = nbytes if nbytes is not None else ts[0].numel() * ts[0].element_size()
    _check(lib().ccube_register_buffers(_ptr_array([t.data_ptr() for t in ts]), n),
           "ccube_register_buffers")


def deregister_buffers(tensors) -> None:
    _check(lib().ccube_deregister_buffers(_ptr_array([t.data_ptr() for t in tensors])),
           "ccube_deregister_buffers")


def allreduce_tree(t, count: Optional[int] = None, stream=None) -> None:
    """In-place tree AllReduce of a contiguous CUDA tensor (nlocal == 1)."""
    if not t.is_contiguous():
        raise CCubeError(ERR_INVALID_ARG, "ccube_allreduce_tree", "tensor must be contiguous")
    n = t.numel() if count is None else count
    _check(lib().ccube_allreduce_tree(t.data_ptr(), n, _dtype_code(t), _stream_handle(stream)),
           "ccube_allreduce_tree")


def allreduce_tree_local(tensors, count: Optional[int] = None, stream=None) -> None:
    """In-place AllReduce over the ranks hosted by this process (loopback)."""
    ts = list(tensors)
    for t in ts:
        if not t.is_contiguous():
            raise CCubeError(ERR_INVALID_ARG, "ccube_allreduce_tree_local",
                             "tensors must be contiguous")
    n = ts[0].numel() if count is None else count
    _check(lib().ccube_allreduce_tree_local(_ptr_array([t.data_ptr() for t in ts]), n,
                                            _dtype_code(ts[0]), _stream_handle(stream)),
           "ccube_allreduce_tree_local")


def allreduce_tree_local_ptrs(ptrs: Sequence[int], count: int, dtype: str, stream) -> None:
    _check(lib().ccube_allreduce_tree_local(_ptr_array(list(ptrs)), count, DTYPE[dtype],
                                            _stream_handle(stream)),
           "ccube_allreduce_tree_local")


def barrier(stream=None) -> None:
    """ccube_barrier: device-side barrier across all ranks, enqueued on ``stream``."""
    _check(lib().ccube_barrier(_stream_handle(stream)), "ccube_barrier")


def plan_launch(P: int, kind: str, nlocal: int, rank: int, nbytes: int, chunk_bytes: int = 0,
                overlap: bool = True, channels: int = 0, cap_ctas: int = 296):
    """ccube_plan_launch (host only): (J, CTAs of rank's process, max CTAs over processes)."""
    j, n, m = ctypes.c_int(), ctypes.c_int(), ctypes.c_int()
    _check(lib().ccube_plan_launch(P, TREE[kind], nlocal, rank, nbytes, chunk_bytes,
                                   1 if overlap else 0, channels, cap_ctas, ctypes.byref(j),
                                   ctypes.byref(n), ctypes.byref(m)), "ccube_plan_launch")
    return j.value, n.value, m.value


def measure_peer_bandwidth(nbytes: int = 64 << 20, iters: int = 5):
    """ccube_measure_peer_bandwidth (collective, one process per GPU): returns
    (pair GB/s as a P x P list, per-GPU egress GB/s for fan-out m = 0..P-1)."""
    P = get_info()["world_size"]
    pair = (ctypes.c_double * (P * P))()
    fan = (ctypes.c_double * P)()
    _check(lib().ccube_measure_peer_bandwidth(nbytes, iters, pair, fan),
           "ccube_measure_peer_bandwidth")
    return [[pair[i * P + j] for j in range(P)] for i in range(P)], list(fan)


# ------------------------------------------------------------------ gradient queue

def gradq_set_layers(layer_end_elems: Sequence[int]) -> None:
    arr = (ctypes.c_size_t * len(layer_end_elems))(*layer_end_elems)
    _check(lib().ccube_gradq_set_layers(arr, len(layer_end_elems)), "ccube_gradq_set_layers")


def gradq_wait(layer_id: int, stream=None) -> None:
    _check(lib().ccube_gradq_wait(layer_id, _stream_handle(stream)), "ccube_gradq_wait")


def gradq_wait_local(local_rank: int, layer_id: int, stream=None) -> None:
    _check(lib().ccube_gradq_wait_local(local_rank, layer_id, _stream_handle(stream)),
           "ccube_gradq_wait_local")


def gradq_set_sgd(weights, alpha: float = 0.0) -> None:
    """Fused SGD update (f2): ``weights`` = one contiguous fp32 CUDA tensor per rank
    hosted by this process (gradient-buffer layout), or None to disable."""
    if weights is None:
        _check(lib().ccube_gradq_set_sgd(None, 0, 0.0), "ccube_gradq_set_sgd")
        return
    ws = list(weights)
    for w in ws:
        if not w.is_contiguous():
            raise CCubeError(ERR_INVALID_ARG, "ccube_gradq_set_sgd", "weights must be contiguous")
    nbytes = min(w.numel() * w.element_size() for w in ws)
    _check(lib().ccube_gradq_set_sgd(_ptr_array([w.data_ptr() for w in ws]), nbytes, alpha),
           "ccube_gradq_set_sgd")


# ------------------------------------------------------------------------- knobs

def set_overlap(on: bool) -> None:
    _check(lib().ccube_set_overlap(1 if on else 0), "ccube_set_overlap")


def set_channels(channels: int) -> None:
    """Channels per tree (0 = auto).  Collective with several processes."""
    _check(lib().ccube_set_channels(channels), "ccube_set_channels")


def set_threads(threads: int) -> None:
    """Data threads per CTA (32..256, multiple of 32), or 0 = auto (the default: 6 data
    warps when the channel slices hold >= 3 units of 2 KB, else 8)."""
    _check(lib().ccube_set_threads(threads), "ccube_set_threads")


def set_transport(mode: str) -> None:
    """'auto' (pull inside a GPU, push across GPUs), 'push' or 'pull'."""
    _check(lib().ccube_set_transport(TRANSPORT[mode]), "ccube_set_transport")


def set_datapath(mode: str) -> None:
    """'auto' (default: TMA for the rotated tree set), 'lsu' (register-staged) or 'tma'
    (cp.async.bulk shared-memory ring)."""
    _check(lib().ccube_set_datapath(DATAPATH[mode]), "ccube_set_datapath")


def set_protocol(ll: bool) -> None:
    """True (default): one-chunk calls run the LL (flag-in-data) kernel; False: the
    chunked kernel for every size.  Same result either way."""
    _check(lib().ccube_set_protocol(1 if ll else 0), "ccube_set_protocol")


def set_trace(trace_tensor, kmax: int) -> None:
    ptr = None if trace_tensor is None else trace_tensor.data_ptr()
    _check(lib().ccube_set_trace(ptr, kmax if ptr else 0), "ccube_set_trace")


def get_info() -> dict:
    info = Info()
    _check(lib().ccube_get_info(ctypes.byref(info)), "ccube_get_info")
    d = {k: getattr(info, k) for k, _ in Info._fields_ if k != "epoch_base"}
    d["epoch_base"] = list(info.epoch_base)
    return d


def tree_parents(P: int, kind: str, tree: int):
    out = (ctypes.c_int * P)()
    _check(lib().ccube_tree_parents(P, TREE[kind], tree, out), "ccube_tree_parents")
    return list(out)


def set_placement(perm: Optional[Sequence[int]]) -> None:
    """Tree position v is hosted by rank perm[v] from the next init on (R19); None
    restores the identity.  Every rank must pass the same permutation."""
    if perm is None:
        _check(lib().ccube_set_placement(None, 0), "ccube_set_placement")
        return
    arr = (ctypes.c_int * len(perm))(*perm)
    _check(lib().ccube_set_placement(arr, len(perm)), "ccube_set_placement")


def plan_placement(bw, kind: str = "double"):
    """Least-cost placement for a P x P peer bandwidth matrix (nested sequences or
    an array; bw[i][j] = rank i -> rank j)."""
    P = len(bw)
    flat = (ctypes.c_double * (P * P))(*[float(bw[i][j]) for i in range(P) for j in range(P)])
    out = (ctypes.c_int * P)()
    _check(lib().ccube_plan_placement(P, TREE[kind], flat, out), "ccube_plan_placement")
    return list(out)


def tree_parents_placed(P: int, kind: str, tree: int, perm: Optional[Sequence[int]]):
    arr = None if perm is None else (ctypes.c_int * P)(*perm)
    out = (ctypes.c_int * P)()
    _check(lib().ccube_tree_parents_placed(P, TREE[kind], tree, arr, out),
           "ccube_tree_parents_placed")
    return list(out)

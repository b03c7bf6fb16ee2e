"""One process per rank (nlocal == 1): CUDA IPC peer mapping, .sys-scope flags and
PUSH edges — the multi-GPU code path — run as 2-4 processes sharing cuda:0
(CCUBE_ALLOW_SHARED_GPU=1; contexts time-slice, so progress is slow but the
protocol is the one that runs across GPUs over NVSwitch).  Bootstrap over gloo.

Bar: every rank bit-exact to the oracle definition (oracle.allreduce.reference),
and the gradient-queue gate opens only after a layer's chunks landed."""

import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, kind, dtype, count, chunk, q, perm=None):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    os.environ["CCUBE_ALLOW_SHARED_GPU"] = "1"
    import torch
    import torch.distributed as dist
    from paper_conf_hpca_sanghoonsk23_b200 import ccube, inputs
    try:
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        ccube.set_placement(perm)
        ccube.init_distributed(dist.group.WORLD, tree=kind, chunk_bytes=chunk)
        ccube.set_channels(2)
        x = inputs.gradients(rank, count, dtype)
        t = (torch.from_numpy(x.view(np.int16)).view(torch.bfloat16) if dtype == "bfloat16"
             else torch.from_numpy(x)).cuda()
        ends = [count // 3, count // 2, count]
        ccube.gradq_set_layers(ends)
        comm, comp = torch.cuda.Stream(), torch.cuda.Stream()
        snaps = []
        for _ in range(2):   # two epochs: counters advance, buffers re-registered once
            t.copy_(torch.from_numpy(x.view(np.int16)).view(torch.bfloat16) if dtype == "bfloat16"
                    else torch.from_numpy(x))
            torch.cuda.synchronize()
            ccube.allreduce_tree(t, stream=comm)
            with torch.cuda.stream(comp):
                snaps = []
                lo = 0
                for l, hi in enumerate(ends):
                    ccube.gradq_wait(l, stream=comp)
                    snaps.append(t[lo:hi].clone())
                    lo = hi
            torch.cuda.synchronize()
        out = t.cpu()
        out = out.view(torch.int16).numpy().view(np.uint16) if dtype == "bfloat16" else out.numpy()
        early = [not torch.equal(s.cpu(), t[lo:hi].cpu())
                 for s, lo, hi in zip(snaps, [0] + ends[:-1], ends)]
        ccube.finalize()
        q.put((rank, "", out, any(early)))
    except Exception as e:  # noqa: BLE001
        q.put((rank, repr(e), None, None))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


def _run(world, kind, dtype, count, chunk, perm=None):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, kind, dtype, count, chunk, q, perm))
             for r in range(world)]
    for p in procs:
        p.start()
    res = sorted((q.get(timeout=300) for _ in procs), key=lambda r: r[0])
    for p in procs:
        p.join(timeout=60)
    return res


@pytest.mark.parametrize("world,kind,dtype", [(2, "single", "float32"),
                                              (4, "rotated", "float32"),
                                              (3, "double", "bfloat16"),
                                              (4, "double", "float32"),
                                              (4, "single", "int32")])
def test_multiprocess_ipc_parity(world, kind, dtype):
    from oracle import allreduce as oar
    from paper_conf_hpca_sanghoonsk23_b200 import inputs
    count, chunk = 50_001, 16 << 10
    res = _run(world, kind, dtype, count, chunk)
    xs = [inputs.gradients(r, count, dtype) for r in range(world)]
    ref = oar.reference(xs, kind, chunk, dtype)[0]
    for rank, err, out, early in res:
        assert err == "", f"rank {rank}: {err}"
        assert np.array_equal(out, ref), f"rank {rank} differs from the oracle"
        assert not early, f"rank {rank}: a gate opened before its layer landed"


def test_multiprocess_ipc_parity_placed():
    """A placed double tree (R19) across processes: bit-exact to the oracle with the
    same permutation (the gradient-queue gates included)."""
    from oracle import allreduce as oar
    from paper_conf_hpca_sanghoonsk23_b200 import inputs
    world, kind, dtype, perm = 4, "double", "float32", [2, 0, 3, 1]
    count, chunk = 50_001, 16 << 10
    res = _run(world, kind, dtype, count, chunk, perm)
    xs = [inputs.gradients(r, count, dtype) for r in range(world)]
    ref = oar.reference(xs, kind, chunk, dtype, perm=perm)[0]
    assert not np.array_equal(ref, oar.reference(xs, kind, chunk, dtype)[0])
    for rank, err, out, early in res:
        assert err == "", f"rank {rank}: {err}"
        assert np.array_equal(out, ref), f"rank {rank} differs from the oracle"
        assert not early, f"rank {rank}: a gate opened before its layer landed"

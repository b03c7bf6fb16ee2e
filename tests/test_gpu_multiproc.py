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


@pytest.mark.parametrize("world,kind,dtype,count", [(2, "single", "float32", 50_001),
                                                    (4, "rotated", "float32", 50_001),
                                                    (3, "double", "bfloat16", 50_001),
                                                    (4, "double", "float32", 50_001),
                                                    (4, "single", "int32", 50_001),
                                                    (4, "double", "float32", 3_001),
                                                    (3, "single", "bfloat16", 4_095)])
def test_multiprocess_ipc_parity(world, kind, dtype, count):
    """The last two cases are one chunk: the LL kernel's remote LL-line stores and
    polls at .sys scope, and its Enqueue Semaphore for the gates."""
    from oracle import allreduce as oar
    from paper_conf_hpca_sanghoonsk23_b200 import inputs
    chunk = 16 << 10
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


# ---- generic spawner for the scenarios below -----------------------------------------

def _scenario_entry(rank, world, port, name, args, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    os.environ["CCUBE_ALLOW_SHARED_GPU"] = "1"
    for k, v in args.get("env", {}).items():
        os.environ[k] = v
    import torch
    import torch.distributed as dist
    try:
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        q.put((rank, "", globals()[name](rank, world, **args.get("kw", {}))))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, repr(e) + traceback.format_exc(), None))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


def _spawn(world, name, **args):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_scenario_entry, args=(r, world, port, name, args, q))
             for r in range(world)]
    for p in procs:
        p.start()
    res = sorted((q.get(timeout=600) for _ in procs), key=lambda r: r[0])
    for p in procs:
        p.join(timeout=60)
    for rank, err, _ in res:
        assert err == "", f"rank {rank}: {err}"
    return [r[2] for r in res]


def _auto_channels(rank, world, kind, dtype, count, chunk, overlap):
    import torch
    import torch.distributed as dist
    from paper_conf_hpca_sanghoonsk23_b200 import ccube, inputs
    ccube.init_distributed(dist.group.WORLD, tree=kind, chunk_bytes=chunk)
    ccube.set_overlap(overlap)          # channels stay 0: auto
    x = inputs.gradients(rank, count, dtype)
    t = torch.from_numpy(x).cuda()
    ccube.allreduce_tree(t)
    torch.cuda.synchronize()
    info = ccube.get_info()
    ccube.finalize()
    return t.cpu().numpy(), info["last_channels"], info["last_ctas"]


@pytest.mark.parametrize("kind,overlap", [("double", True), ("double", False),
                                          ("single", True)])
def test_multiprocess_auto_channels_many_chunks(kind, overlap):
    """one process per rank with AUTO channels and >= 16 chunks of
    256 KiB, where the round-1 per-process rule gave the roots of the double tree a
    different J than the other ranks (and hung).  Every rank must pick the same J,
    and the result must be bit-exact to the oracle."""
    from oracle import allreduce as oar
    from paper_conf_hpca_sanghoonsk23_b200 import ccube, inputs
    world, dtype, chunk = 4, "float32", 256 << 10
    count = 17 * (chunk // 4) + 123
    out = _spawn(world, "_auto_channels", kw=dict(kind=kind, dtype=dtype, count=count,
                                                  chunk=chunk, overlap=overlap))
    xs = [inputs.gradients(r, count, dtype) for r in range(world)]
    ref = oar.reference(xs, kind, chunk, dtype)[0]
    Js = {J for _, J, _ in out}
    assert len(Js) == 1, out
    # the library's host-side plan (cap from the real occupancy) names the same J
    # for every rank; here it must be > 64, i.e. the cap, not the unit limit, binds
    assert Js.pop() > 64
    for rank, (res, _, _) in enumerate(out):
        assert np.array_equal(res, ref), f"rank {rank}"


def _setting_mismatch(rank, world):
    import torch.distributed as dist
    from paper_conf_hpca_sanghoonsk23_b200 import ccube
    ccube.init_distributed(dist.group.WORLD, tree="double", chunk_bytes=64 << 10)
    codes = []
    for fn, args in [(ccube.set_channels, (4 + 4 * rank,)),   # differ
                     (ccube.set_channels, (6,)),              # agree
                     (ccube.set_overlap, (rank == 0,)),       # differ
                     (ccube.set_threads, (rank * 1000 + 32,)),  # rank 1's is invalid
                     (ccube.set_datapath, ("lsu",))]:         # agree
        try:
            fn(*args)
            codes.append(0)
        except ccube.CCubeError as e:
            codes.append(e.code)
    info = ccube.get_info()
    ccube.finalize()
    return codes, info["channels"], info["threads"]


def test_multiprocess_settings_are_collective():
    """a setting one rank changes differently is refused on EVERY
    rank (INVALID_ARG), so no rank launches with a slicing its peers do not share."""
    from paper_conf_hpca_sanghoonsk23_b200 import ccube
    out = _spawn(2, "_setting_mismatch")
    bad = ccube.ERR_INVALID_ARG
    for codes, channels, threads in out:
        assert codes == [bad, 0, bad, bad, 0], codes
        assert channels == 6 and threads == 0   # auto, the default (rank 1 passed an invalid value)


def _watchdog(rank, world):
    import torch
    import torch.distributed as dist
    from paper_conf_hpca_sanghoonsk23_b200 import ccube
    pg = dist.group.WORLD
    ccube.init_distributed(pg, tree="single", chunk_bytes=16 << 10)
    t = torch.ones(100_000, device="cuda") * (rank + 1)
    ccube.register_buffers([t])
    codes = []
    if rank == 0:          # rank 1 never joins this AllReduce
        ccube.allreduce_tree(t)
        torch.cuda.synchronize()
        try:
            ccube.allreduce_tree(t)
            codes.append(0)
        except ccube.CCubeError as e:
            codes.append(e.code)
            codes.append("watchdog" in str(e))
    dist.barrier()
    ccube.finalize()       # collective, also on the poisoned rank
    # a fresh communicator works again
    ccube.init_distributed(pg, tree="single", chunk_bytes=16 << 10)
    t.fill_(rank + 1)
    ccube.allreduce_tree(t)
    torch.cuda.synchronize()
    ok = bool((t == 3).all().item())
    ccube.finalize()
    return codes, ok


def test_watchdog_timeout_then_reinit():
    """a7's watchdog (SURVEY §4 layer 2): a rank that never calls makes its peer's
    kernel abort after CCUBE_WATCHDOG_MS; the next call returns CCUBE_ERR_TIMEOUT,
    finalize still works, and a fresh init runs a correct AllReduce."""
    from paper_conf_hpca_sanghoonsk23_b200 import ccube
    out = _spawn(2, "_watchdog", env={"CCUBE_WATCHDOG_MS": "1500"})
    assert out[0] == ([ccube.ERR_TIMEOUT, True], True), out[0]
    assert out[1] == ([], True), out[1]


def _barrier(rank, world, sleep_ms):
    import torch
    import torch.distributed as dist
    from paper_conf_hpca_sanghoonsk23_b200 import ccube
    ccube.init_distributed(dist.group.WORLD, tree="double", chunk_bytes=16 << 10)
    s = torch.cuda.Stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    dist.barrier()
    with torch.cuda.stream(s):
        if rank == world - 1:   # the last rank arrives late
            torch.cuda._sleep(int(sleep_ms * 1.9e6))
        e0.record(s)
        ccube.barrier(s)
        e1.record(s)
        for _ in range(3):
            ccube.barrier(s)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    ccube.finalize()
    return ms


def test_device_barrier_waits_for_the_last_rank():
    """ccube_barrier (bench.py's start barrier): no rank leaves before the last one
    arrived; rank 0's wait covers the late rank's ~200 ms delay."""
    out = _spawn(3, "_barrier", kw=dict(sleep_ms=200))
    assert out[0] >= 150, out


def _peer_bw(rank, world):
    import torch.distributed as dist
    from paper_conf_hpca_sanghoonsk23_b200 import ccube
    ccube.init_distributed(dist.group.WORLD, tree="double", chunk_bytes=64 << 10)
    pair, fan = ccube.measure_peer_bandwidth(4 << 20, 2)
    t = __import__("torch").ones(1000, device="cuda") * (rank + 1)
    ccube.allreduce_tree(t)     # the communicator still works afterwards
    __import__("torch").cuda.synchronize()
    ok = bool((t == world * (world + 1) / 2).all().item())
    ccube.finalize()
    return pair, fan, ok


def test_measure_peer_bandwidth_runs_collectively():
    """The NVLink roofline instrument's plumbing (IPC mapping of every peer, device
    barrier, device timing, the exchange): every rank gets the same P x P matrix with
    positive off-diagonal entries.  On one shared GPU the numbers are local copies,
    not NVLink figures."""
    out = _spawn(3, "_peer_bw")
    pair0, fan0, _ = out[0]
    for pair, fan, ok in out:
        assert pair == pair0 and fan == fan0 and ok
    for i in range(3):
        for j in range(3):
            assert (pair0[i][j] > 0) == (i != j)
    assert fan0[0] == 0 and all(f > 0 for f in fan0[1:])


@pytest.mark.parametrize("kind,count", [("double", 70_001), ("single", 3_001)])
def test_multiprocess_ipc_parity_p8(kind, count):
    """Eight processes (the target's P): the double tree chunked (16 KiB chunks,
    interior ranks in one tree and leaves in the other, every edge PUSH over IPC)
    and a one-chunk message on the LL kernel, bit-exact to the oracle with the
    gates checked, as in test_multiprocess_ipc_parity."""
    from oracle import allreduce as oar
    from paper_conf_hpca_sanghoonsk23_b200 import inputs
    world, dtype, chunk = 8, "float32", 16 << 10
    res = _run(world, kind, dtype, count, chunk)
    xs = [inputs.gradients(r, count, dtype) for r in range(world)]
    ref = oar.reference(xs, kind, chunk, dtype)[0]
    for rank, err, out, early in res:
        assert err == "", f"rank {rank}: {err}"
        assert np.array_equal(out, ref), f"rank {rank} differs from the oracle"
        assert not early, f"rank {rank}: a gate opened before its layer landed"


@pytest.mark.parametrize("world,kind", [(4, "double"), (3, "single"), (4, "rotated")])
def test_multiprocess_pull_transport(monkeypatch, world, kind):
    """Every edge PULL across processes (CCUBE_TRANSPORT=2): a parent reads its
    children's partials in place over IPC, so each leaf process runs its pulled
    leaves on its leaf-group CTA (heads published at once, results awaited at .sys
    scope).  Bit-exact vs the oracle, gates included."""
    from oracle import allreduce as oar
    from paper_conf_hpca_sanghoonsk23_b200 import inputs
    monkeypatch.setenv("CCUBE_TRANSPORT", "2")
    dtype, count, chunk = "float32", 50_001, 16 << 10
    res = _run(world, kind, dtype, count, chunk)
    xs = [inputs.gradients(r, count, dtype) for r in range(world)]
    ref = oar.reference(xs, kind, chunk, dtype)[0]
    for rank, err, out, early in res:
        assert err == "", f"rank {rank}: {err}"
        assert np.array_equal(out, ref), f"rank {rank} differs from the oracle"
        assert not early, f"rank {rank}: a gate opened before its layer landed"

#!/usr/bin/env python3
"""C-Cube bench: tree AllReduce bus bandwidth on B200 (BASELINE.json metric).

N=1 (default): the workload of BASELINE.json configs[1] — the ResNet-50 gradient
set (25,557,032 fp32, 102,228,128 B per rank) — reduced across P=8 logical ranks
hosted on ONE B200 ("loopback": the same kernel body that runs one process per
GPU; every rank's buffer lives in local HBM).  One step = one
ccube_allreduce_tree_local call = one kernel launch = the whole hot path (a3-a8:
chunking, reduce-up, C1 turnaround, broadcast-down, enqueue semaphores).

N>1 (torchrun, one process per GPU): P = N real ranks, each with its own
102 MB buffer, peers mapped over NVLink/NVSwitch with CUDA IPC.

busbw = algbw * 2(P-1)/P with algbw = bytes_per_rank / t (nccl-tests
convention), t = device time (CUDA events on the launching stream; max over
ranks for N>1).  --impl reference times the CPU oracle (oracle/) instead.
"""

import argparse
import json
import os
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "AllReduce busbw GB/s vs size at 2/4/8 B200 (% of 900 GB/s); iter time chained vs unchained"
NVLINK_NOMINAL_GBS = 900.0
NVLINK_MEASURED_GBS = 770.0   # B200_PROFILING.md: measured peer copy per direction


def parse(argv=None):
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=200)
    p.add_argument("--warmup", type=int, default=10)
    p.add_argument("--impl", choices=["ccube", "reference"], default="ccube")
    p.add_argument("--workload", choices=["resnet50", "vgg16"], default="resnet50")
    p.add_argument("--dtype", choices=["float32", "bfloat16", "int32"], default=None)
    p.add_argument("--tree", choices=["single", "double", "rotated"], default=None)
    p.add_argument("--ranks", type=int, default=8, help="logical ranks in loopback (N=1)")
    p.add_argument("--overlap", type=int, default=1, help="1 = C1, 0 = B")
    p.add_argument("--chunk-bytes", type=int, default=256 << 10)
    p.add_argument("--channels", type=int, default=0)
    p.add_argument("--threads", type=int, default=0)
    p.add_argument("--datapath", choices=["auto", "tma", "lsu"], default=None,
                   help="data-warp datapath (default: the library's, CCUBE_DATAPATH)")
    p.add_argument("--e2e-steps", type=int, default=10)
    p.add_argument("--e2e-copy-streams", type=int, default=1,
                   help="e2e: streams (copy engines) per copy direction")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-clocks", action="store_true")
    p.add_argument("--no-nccl", action="store_true",
                   help="N>1: skip the NCCL Ring/Tree/default comparison on the same buffer")
    p.add_argument("--nccl-steps", type=int, default=20)
    p.add_argument("--max-elems", type=int, default=0,
                   help="test runs only: time a prefix of the workload (0 = all of it)")
    p.add_argument("--plan-placement", action="store_true",
                   help="N>1: measure peer bandwidth and place the trees on it (R19)")
    p.add_argument("--cpu-seconds", type=float, default=10.0,
                   help="cpu_baseline: repeat the oracle sample until this much CPU work")
    p.add_argument("--cpu-sample-chunks", type=int, default=0,
                   help="chunks per step for the oracle (0 = auto)")
    p.add_argument("--mode", choices=["allreduce", "iter"], default="allreduce",
                   help="iter: only the chained-vs-unchained training iteration")
    p.add_argument("--no-iter", action="store_true",
                   help="skip the chained-iteration sub-benchmark in the default line")
    p.add_argument("--iter-batch", type=int, default=64)
    p.add_argument("--iter-model", choices=["resnet50", "vgg16", "zfnet"], default="resnet50")
    p.add_argument("--iter-fused-sgd", action="store_true",
                   help="apply the SGD step inside the AllReduce kernel (f2)")
    p.add_argument("--iter-steps", type=int, default=20)
    p.add_argument("--iter-rounds", type=int, default=5)
    p.add_argument("--iter-warmup", type=int, default=2)
    p.add_argument("--iter-channels", type=int, default=4,
                   help="loopback: AllReduce channels of the chained iteration")
    p.add_argument("--iter-channels-multi", type=int, default=16,
                   help="N>1: AllReduce channels of the chained iteration (0 = auto, which "
                        "gives the AllReduce every SM and the forward nothing to overlap on)")
    p.add_argument("--iter-tree", choices=["single", "double", "rotated"], default="single")
    p.add_argument("--iter-rank", type=int, default=1,
                   help="loopback rank that hosts the model replica (1 = a leaf of tree 0)")
    p.add_argument("--no-port-peak", action="store_true",
                   help="N>1: skip the peer-store bandwidth probe (roofline peak)")
    p.add_argument("--no-extra", action="store_true",
                   help="skip the other tree kinds and the VGG-16 bf16 double-tree line")
    p.add_argument("--extra-steps", type=int, default=20)
    p.add_argument("--cpu-cores", type=int, default=0,
                   help="cpu_baseline: also time the oracle on this many host cores "
                        "(0 = all of them, 1 = skip the all-cores figure)")
    a = p.parse_args(argv)
    if a.dtype is None:
        a.dtype = "bfloat16" if a.workload == "vgg16" else "float32"
    if a.tree is None:
        a.tree = "double" if a.workload == "vgg16" else "single"
    return a


def parse_args_list(argv):
    """parse() on an explicit argument list (tools reuse bench.py's defaults)."""
    return parse(argv)


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    except Exception:  # noqa: BLE001
        return 6650.0, "fallback (B200_PROFILING.md)"


# ------------------------------------------------------------------------ clocks
class ClockSampler:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device_index=0, enabled=True):
        self.proc = None
        self.path = os.path.join("/tmp", f"ccube_clocks_{os.getpid()}.csv")
        self.dev = device_index
        if enabled:
            try:
                self.proc = subprocess.Popen(
                    ["nvidia-smi", "-i", str(device_index), f"--query-gpu={self.FIELDS}",
                     "--format=csv,noheader,nounits", "-lms", "100"],
                    stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
            except Exception:  # noqa: BLE001
                self.proc = None

    def stop(self):
        if self.proc is None:
            return None
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:  # noqa: BLE001
            self.proc.kill()
        rows = []
        for line in open(self.path):
            parts = [x.strip() for x in line.split(",")]
            if len(parts) < 9:
                continue
            try:
                rows.append(parts)
            except Exception:  # noqa: BLE001
                pass
        if not rows:
            return None
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        smax = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4)
                          if r[5 + i].lower().startswith("active")})
        return {"sm_mhz": float(np.median(sm)) if sm else None,
                "sm_max_mhz": max(smax) if smax else None,
                "reasons": reasons, "samples": len(rows)}


# ------------------------------------------------------------- NVLink counters
class NvlinkCounters:
    """NVLink data bytes this GPU sent / received, from NVML's cumulative per-link
    counters (NVML_FI_DEV_NVLINK_THROUGHPUT_DATA_TX / _RX, KiB; summed over links).
    Read before and after the timed region at N > 1; unlike an ncu pass it does not
    serialise the ranks' kernels.  Any failure (no NVML, no NVLink) gives None."""

    LINKS = 18   # NVLink 5 links per B200

    def __init__(self, device_index):
        self.h = None
        try:
            import pynvml as nv
            import torch
            nv.nvmlInit()
            pr = torch.cuda.get_device_properties(device_index)
            bus = f"{pr.pci_domain_id:08x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
            try:
                self.h = nv.nvmlDeviceGetHandleByPciBusId_v2(bus.encode())
            except Exception:  # noqa: BLE001
                self.h = nv.nvmlDeviceGetHandleByIndex(device_index)
            self.nv = nv
        except Exception:  # noqa: BLE001
            self.h = None

    def read(self):
        """(tx_bytes, rx_bytes) cumulative, or None."""
        if self.h is None:
            return None
        nv = self.nv
        try:
            ids = [(nv.NVML_FI_DEV_NVLINK_THROUGHPUT_DATA_TX, l) for l in range(self.LINKS)] + \
                  [(nv.NVML_FI_DEV_NVLINK_THROUGHPUT_DATA_RX, l) for l in range(self.LINKS)]
            vals = nv.nvmlDeviceGetFieldValues(self.h, ids)
            tx = sum(v.value.ullVal for v in vals[:self.LINKS] if v.nvmlReturn == 0)
            rx = sum(v.value.ullVal for v in vals[self.LINKS:] if v.nvmlReturn == 0)
            return tx * 1024, rx * 1024
        except Exception:  # noqa: BLE001
            return None


# ---------------------------------------------------------------- oracle timing
def oracle_inputs(P, dtype, workload, chunk_bytes, nchunks):
    """Every rank's seeded gradients for the first ``nchunks`` chunks of the workload."""
    from oracle import arith
    from paper_conf_hpca_sanghoonsk23_b200 import inputs, workloads
    ends = workloads.layer_ends(workload)
    E = chunk_bytes // arith.ELEM_SIZE[dtype]
    count = min(ends[-1], nchunks * E)
    xs = [inputs.gradients(r, ends[-1], dtype, layer_ends=ends, lo=0, hi=count) for r in range(P)]
    return xs, count * arith.ELEM_SIZE[dtype]


def oracle_replay_time(xs, tree, dtype, chunk_bytes, overlap):
    """(seconds, root's result) for one run of the CPU oracle's message-passing replay."""
    from oracle import allreduce as oar
    t0 = time.perf_counter()
    out, _ = oar.replay(xs, tree, chunk_bytes, dtype, overlap=bool(overlap))
    return time.perf_counter() - t0, out[0]


def oracle_time(P, tree, dtype, workload, chunk_bytes, nchunks, overlap, min_seconds=0.0,
                max_reps=64):
    """Time the CPU oracle's replay on the first ``nchunks`` chunks of the workload
    (every rank's data for those chunks), repeated until at least ``min_seconds`` of
    CPU work (at most ``max_reps`` replays).  Returns (seconds per replay, bytes per
    rank per replay, replays, the oracle's result for those elements)."""
    xs, nbytes = oracle_inputs(P, dtype, workload, chunk_bytes, nchunks)
    reps, total, res = 0, 0.0, None
    while reps == 0 or (total < min_seconds and reps < max_reps):
        dt, res = oracle_replay_time(xs, tree, dtype, chunk_bytes, overlap)
        total += dt
        reps += 1
    return total / reps, nbytes, reps, res


def _oracle_worker(args):
    """One host core's share of the all-cores oracle run: the replay of chunks
    [c0, c1) (c0 a multiple of the tree count, so chunk c keeps tree c mod T)."""
    from multiprocessing import shared_memory
    name, shape, npdt, tree, dtype, chunk_bytes, overlap, c0, c1, reps = args
    shm = shared_memory.SharedMemory(name=name)
    try:
        allx = np.ndarray(shape, dtype=npdt, buffer=shm.buf)
        E = chunk_bytes // allx.itemsize
        xs = [allx[r, c0 * E:min(c1 * E, shape[1])] for r in range(shape[0])]
        t0 = time.perf_counter()
        for _ in range(reps):
            oracle_replay_time(xs, tree, dtype, chunk_bytes, overlap)
        return time.perf_counter() - t0
    finally:
        shm.close()


def _cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


class OraclePool:
    """The oracle as it stands on ALL host cores: the sample's chunks
    are split into one contiguous range per core (ranges start at multiples of the
    tree count, so the tree of every chunk is unchanged) and each core replays its
    range in its own process; ``run`` returns the wall time of one pass of the pool.
    The sample is ``nchunks_per_core`` x cores chunks, capped at the workload."""

    def __init__(self, P, tree, dtype, workload, chunk_bytes, nchunks_per_core, overlap,
                 cores=0, xs_full=None):
        import multiprocessing as mp
        from multiprocessing import shared_memory
        from oracle import arith
        from paper_conf_hpca_sanghoonsk23_b200 import workloads
        self.P, self.tree, self.workload = P, tree, workload
        cores = cores or len(os.sched_getaffinity(0))
        T = {"single": 1, "double": 2, "rotated": P}[tree]
        E = chunk_bytes // arith.ELEM_SIZE[dtype]
        K = -(-workloads.layer_ends(workload)[-1] // E)
        self.nch = min(K, nchunks_per_core * cores)
        if xs_full is not None:   # every rank's whole input, already generated
            n = min(xs_full[0].size, self.nch * E)
            xs, self.nbytes = [x[:n] for x in xs_full], n * arith.ELEM_SIZE[dtype]
        else:
            xs, self.nbytes = oracle_inputs(P, dtype, workload, chunk_bytes, self.nch)
        per = -(-self.nch // cores)
        per = -(-per // T) * T
        ranges = [(c0, min(self.nch, c0 + per)) for c0 in range(0, self.nch, per)]
        self.cores = len(ranges)
        self.shm = shared_memory.SharedMemory(create=True, size=xs[0].nbytes * P)
        allx = np.ndarray((P, xs[0].size), dtype=xs[0].dtype, buffer=self.shm.buf)
        for r in range(P):
            allx[r] = xs[r]
        self.args = [(self.shm.name, allx.shape, allx.dtype, tree, dtype, chunk_bytes, overlap,
                      c0, c1, 1) for c0, c1 in ranges]
        self.pool = mp.get_context("spawn").Pool(self.cores)
        self.pool.map(_oracle_worker, self.args)          # warm-up (imports, pages)
        self.busy = 0.0

    def run(self, reps=1):
        args = [x[:-1] + (reps,) for x in self.args]
        t0 = time.perf_counter()
        self.busy += sum(self.pool.map(_oracle_worker, args))
        return (time.perf_counter() - t0) / reps

    def describe(self, passes):
        return (f"oracle.allreduce.replay on the first {self.nch} chunks ({self.nbytes} B per "
                f"rank) of the {self.workload} gradient set, P={self.P}, {self.tree} tree, split "
                f"into {self.cores} chunk ranges, one process per host core; wall time of the "
                f"pool, {passes} passes ({self.busy:.1f} s of CPU work)")

    def close(self):
        self.pool.close()
        self.pool.join()
        self.shm.close()
        self.shm.unlink()


def oracle_time_parallel(P, tree, dtype, workload, chunk_bytes, nchunks_per_core, overlap,
                         cores=0, min_cpu_seconds=10.0, max_passes=200, xs_full=None):
    """The all-cores figure: passes of the pool until ``min_cpu_seconds`` of CPU work
    (summed over the cores) were spent; mean wall time per pass."""
    pool = OraclePool(P, tree, dtype, workload, chunk_bytes, nchunks_per_core, overlap, cores,
                      xs_full)
    try:
        walls = []
        while not walls or (pool.busy < min_cpu_seconds and len(walls) < max_passes):
            walls.append(pool.run())
        wall = float(np.mean(walls))
        bw, _ = busbw(pool.nbytes, wall, P)
        return {"value": bw, "unit": "GB/s", "cores": pool.cores, "kind": "oracle",
                "nproc": len(os.sched_getaffinity(0)), "cpu_model": _cpu_model(),
                "sample": pool.describe(len(walls) + 1), "seconds_per_pass": wall}
    finally:
        pool.close()


def busbw(bytes_per_rank, seconds, P):
    alg = bytes_per_rank / seconds / 1e9
    return alg * 2 * (P - 1) / P, alg


def run_reference(a):
    """--impl reference: the CPU oracle as it stands, on the host cores (rank 0 only).
    One step = one pass of the oracle's replay over the sample, split over every
    host core (--cpu-cores 0, default) or on one core (--cpu-cores 1)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    P = a.ranks if a.gpus == 1 else a.gpus
    if a.cpu_cores == 1:
        nchunks = a.cpu_sample_chunks or 128  # 128 chunks x 256 KiB = 32 MiB per rank
        xs, nbytes = oracle_inputs(P, a.dtype, a.workload, a.chunk_bytes, nchunks)
        for _ in range(a.warmup):
            oracle_replay_time(xs, a.tree, a.dtype, a.chunk_bytes, a.overlap)
        total = 0.0
        for _ in range(a.steps):
            total += oracle_replay_time(xs, a.tree, a.dtype, a.chunk_bytes, a.overlap)[0]
        cores = 1
        sample = (f"oracle.allreduce.replay on the first {nchunks} chunks ({nbytes} B per rank) "
                  f"of the {a.workload} gradient set, P={P}, {a.tree} tree, one step = one "
                  f"replay on one core")
    else:
        pool = OraclePool(P, a.tree, a.dtype, a.workload, a.chunk_bytes,
                          a.cpu_sample_chunks or 32, a.overlap, a.cpu_cores)
        try:
            for _ in range(a.warmup):
                pool.run()
            total = sum(pool.run() for _ in range(a.steps))
            nbytes, cores = pool.nbytes, pool.cores
            sample = pool.describe(a.warmup + a.steps) + "; one step = one pass"
        finally:
            pool.close()
    bw, alg = busbw(nbytes, total / a.steps, P)
    line = {
        "impl": "reference", "metric": METRIC, "value": bw, "unit": "GB/s", "n_gpus": a.gpus,
        "steps": a.steps, "warmup": a.warmup, "ms_per_step": total / a.steps * 1e3,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": _dt(a.dtype),
        "data": "synthetic", "config": _config(a, P, nbytes),
        "cpu_baseline": {"value": bw, "unit": "GB/s", "cores": cores, "kind": "oracle",
                         "sample": sample, "nproc": len(os.sched_getaffinity(0)),
                         "cpu_model": _cpu_model()},
        "e2e": {"value": bw, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "algbw": alg,
    }
    print(json.dumps(line), flush=True)


def _dt(d):
    return {"float32": "f32", "bfloat16": "bf16", "int32": "i32"}[d]


def _config(a, P, bytes_per_rank):
    return {"workload": f"{a.workload} gradient set, {a.tree} tree, {'C1' if a.overlap else 'B'}"
                        f", P={P}" + (" logical ranks on 1 GPU (loopback)" if a.gpus == 1 else ""),
            "P": P, "tree": a.tree, "mode": "C1" if a.overlap else "B",
            "chunk_bytes": a.chunk_bytes, "bytes_per_rank": bytes_per_rank,
            "seed": 20230225}


# -------------------------------------------------------------------- GPU arm
def _time_steps(step, restore, steps, warmup, stream, multi, dev):
    """W untimed warm-up steps, then K steps, each restored from the pristine copy
    (flushes L2) and bracketed by CUDA events on the launching stream.  With several
    processes every step starts after ccube_barrier (device-side, same stream) and
    the region is bracketed by a host barrier + synchronize on both sides.  Returns
    (per-step ms on this rank, total ms = max over ranks)."""
    import torch
    import torch.distributed as dist
    from paper_conf_hpca_sanghoonsk23_b200 import ccube
    for _ in range(max(3, warmup)):
        restore()
        if multi:
            ccube.barrier(stream)
        step()
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
           for _ in range(steps)]
    if multi:
        dist.barrier()
    torch.cuda.synchronize()
    for i in range(steps):
        restore()
        if multi:
            ccube.barrier(stream)      # device-side start barrier
        evs[i][0].record(stream)
        step()
        evs[i][1].record(stream)
    torch.cuda.synchronize()
    if multi:
        dist.barrier()
    ms = [s_.elapsed_time(e_) for s_, e_ in evs]
    total = float(np.sum(ms))
    if multi:
        total = _allmax(total, dev)
    return ms, total


def _result_hash(t):
    """Two int64 checksums of a buffer's bits (plain and position-weighted), so that
    any differing or displaced element changes the pair."""
    import torch
    v = (t.view(torch.int32) if t.element_size() == 4 else t.view(torch.int16)).to(torch.int64)
    w = torch.arange(v.numel(), device=v.device, dtype=torch.int64) % 65521 + 1
    return [int(v.sum().item()), int((v * w).sum().item())]


def _ranks_identical(bufs, multi, dev):
    """Loopback: every rank's buffer equal to rank 0's.  One process per GPU: the
    checksums of every rank's result, allgathered and compared."""
    import torch
    import torch.distributed as dist
    if not multi:
        return all(torch.equal(b, bufs[0]) for b in bufs[1:]), None
    h = torch.tensor(_result_hash(bufs[0]), dtype=torch.int64, device=dev)
    out = [torch.empty_like(h) for _ in range(dist.get_world_size())]
    dist.all_gather(out, h)
    hs = [o.cpu().tolist() for o in out]
    return all(x == hs[0] for x in hs), hs


def run_ccube(a):
    import torch
    import torch.distributed as dist
    from paper_conf_hpca_sanghoonsk23_b200 import ccube, inputs, workloads

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    multi = world > 1
    # test mode for the N>1 path on a one-GPU box: every rank on cuda:0 (with
    # CCUBE_ALLOW_SHARED_GPU=1), gloo for the host plumbing, no NCCL comparison
    shared = multi and os.environ.get("CCUBE_BENCH_SHARED_GPU") == "1"
    torch.cuda.set_device(local_rank if multi and not shared else 0)
    dev = torch.device("cuda", torch.cuda.current_device())
    if multi:
        if shared:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
    hdev = None if shared else dev      # where host-side collectives of floats run
    P = world if multi else a.ranks
    nloc = 1 if multi else P

    ends = workloads.layer_ends(a.workload)
    if a.max_elems:   # test runs only: a prefix of the workload
        ends = [min(e, a.max_elems) for e in ends]
    count = ends[-1]
    tdt = {"float32": torch.float32, "bfloat16": torch.bfloat16, "int32": torch.int32}[a.dtype]
    es = torch.tensor([], dtype=tdt).element_size()
    nbytes = count * es

    # inputs: seeded synthetic gradients, generated on the host once, resident in HBM
    my_ranks = [rank] if multi else list(range(P))
    host = []
    for r in my_ranks:
        h = torch.empty(count, dtype=tdt).pin_memory()
        blk = 1 << 24
        for lo in range(0, count, blk):
            hi = min(count, lo + blk)
            x = inputs.gradients(r, count, a.dtype, layer_ends=ends, lo=lo, hi=hi)
            t = torch.from_numpy(x.view(np.int16)).view(torch.bfloat16) if a.dtype == "bfloat16" \
                else torch.from_numpy(x)
            h[lo:hi].copy_(t)
        host.append(h)
    pristine = [h.to(dev) for h in host]
    bufs = [p.clone() for p in pristine]

    placement_info = None
    if multi and a.plan_placement:   # R19: measured peer bandwidth -> tree placement
        from paper_conf_hpca_sanghoonsk23_b200 import placement
        perm, pbw = placement.plan(dist.group.WORLD, kind=a.tree)
        ccube.set_placement(perm)
        placement_info = {"perm": perm, "peer_gbs": pbw}

    def init(kind):
        if multi:
            ccube.init_distributed(dist.group.WORLD, tree=kind, chunk_bytes=a.chunk_bytes)
        else:
            ccube.init_loopback(P, kind, a.chunk_bytes)
        if a.channels:
            ccube.set_channels(a.channels)
        if a.threads:
            ccube.set_threads(a.threads)
        if a.datapath:
            ccube.set_datapath(a.datapath)
        ccube.set_overlap(bool(a.overlap))

    init(a.tree)
    stream = torch.cuda.Stream()

    def allreduce(bs):
        if multi:
            ccube.allreduce_tree(bs[0], stream=stream)
        else:
            ccube.allreduce_tree_local(bs, stream=stream)

    def restorer(bs, ps):
        def restore():
            with torch.cuda.stream(stream):
                for b, p in zip(bs, ps):
                    b.copy_(p)   # loopback: P x bytes > L2 (126 MB), flushes L2
        return restore

    clocks = ClockSampler(local_rank if multi else 0, enabled=(rank == 0 and not a.no_clocks))
    nvl = NvlinkCounters(torch.cuda.current_device()) if multi else None
    time.sleep(0.3)
    nvl0, t_nvl0 = (nvl.read(), time.perf_counter()) if nvl else (None, 0)
    ms, total_ms = _time_steps(lambda: allreduce(bufs), restorer(bufs, pristine), a.steps,
                               a.warmup, stream, multi, hdev)
    nvl1, t_nvl1 = (nvl.read(), time.perf_counter()) if nvl else (None, 0)
    clk = clocks.stop()
    nvlink = None
    if nvl0 is not None and nvl1 is not None:
        # the reads bracket the warm-up and the timed steps: one AllReduce each (the
        # restore copies are local, so every NVLink byte is the AllReduce's)
        calls = a.steps + max(3, a.warmup)
        tx, rx = (nvl1[0] - nvl0[0]) / calls, (nvl1[1] - nvl0[1]) / calls
        t_call = total_ms / a.steps / 1e3
        nvlink = {"tx_bytes_per_call": tx, "rx_bytes_per_call": rx,
                  "tx_gbs": tx / t_call / 1e9, "rx_gbs": rx / t_call / 1e9,
                  "algorithmic_port_bytes": max(_port_loads(P, a.tree)) * nbytes,
                  "source": "NVML NVLINK_THROUGHPUT_DATA_TX/RX of rank 0's GPU, summed over "
                            "links, read around warm-up + timed steps; GB/s = bytes per call / "
                            "device time per call"}
    ms_step = total_ms / a.steps
    bw, alg = busbw(nbytes, ms_step / 1e3, P)

    # correctness of the timed configuration: every rank holds the same result
    ok, hashes = _ranks_identical(bufs, multi, None if shared else dev)
    nchk = min(count, (a.cpu_sample_chunks or 128) * (a.chunk_bytes // es))
    result_prefix = bufs[0][:nchk].cpu() if rank == 0 else None

    # ---- e2e: host buffers -> device -> allreduce -> host, through the public API.
    # Every step copies its inputs in from pinned host memory and its results out.
    # Two device buffer sets alternate so that step i's device->host copy (second
    # stream, the other copy engine) overlaps step i+1's host->device copy.
    e2e = None
    if not a.no_e2e:
        outs = [torch.empty_like(h).pin_memory() for h in host]
        sets = [bufs, [torch.empty_like(b) for b in bufs]]
        ev = lambda: torch.cuda.Event()  # noqa: E731
        # the copies of one direction are spread over `ncs` streams (copy engines); the
        # AllReduce runs on `stream` after every H2D stream of its step
        ncs = max(1, min(a.e2e_copy_streams, len(host)))
        h2d = [stream] + [torch.cuda.Stream() for _ in range(ncs - 1)]
        d2h = [torch.cuda.Stream() for _ in range(ncs)]
        d2h_done = [None, None]

        def e2e_step(i):
            s_ = i % 2
            for q, hs in enumerate(h2d):
                if d2h_done[s_] is not None:      # step i-2's results are out of this set
                    for e_ in d2h_done[s_]:
                        hs.wait_event(e_)
                with torch.cuda.stream(hs):
                    for r in range(q, len(host), ncs):
                        sets[s_][r].copy_(host[r], non_blocking=True)
                if q:
                    e_ = ev()
                    e_.record(hs)
                    stream.wait_event(e_)
            allreduce(sets[s_])
            k = ev()
            k.record(stream)
            d2h_done[s_] = []
            for q, ds in enumerate(d2h):
                ds.wait_event(k)
                with torch.cuda.stream(ds):
                    for r in range(q, len(host), ncs):
                        outs[r].copy_(sets[s_][r], non_blocking=True)
                d2h_done[s_].append(ev())
                d2h_done[s_][-1].record(ds)

        for i in range(2):
            e2e_step(i)
        torch.cuda.synchronize()
        if multi:
            dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for i in range(a.e2e_steps):
            e2e_step(i)
        for ds in d2h:
            stream.wait_stream(ds)
        e1.record(stream)
        torch.cuda.synchronize()
        e2e_ms = e0.elapsed_time(e1) / a.e2e_steps
        if multi:
            e2e_ms = _allmax(e2e_ms, hdev)
        ebw, _ = busbw(nbytes, e2e_ms / 1e3, P)
        ok_e2e = all(torch.equal(o, outs[0]) for o in outs[1:]) if not multi else None
        e2e = {"value": ebw, "unit": "GB/s", "ms_per_step": e2e_ms,
               "h2d_bytes_per_step": nbytes * len(my_ranks),
               "d2h_bytes_per_step": nbytes * len(my_ranks), "steps": a.e2e_steps,
               "pipelining": f"two device buffer sets; step i's D2H overlaps step i+1's H2D; "
                             f"each direction on {ncs} stream(s)",
               "ranks_identical": ok_e2e}
        del sets

    # ---- NVLink roofline instrument (N>1): the kernel's own peer-store path
    port_peak = None
    if multi and not a.no_port_peak:
        try:
            pair, fan = ccube.measure_peer_bandwidth(64 << 20, 5)
        except Exception as e:  # noqa: BLE001 — reported; the roofline falls back
            pair, fan = None, None
            port_peak = {"error": repr(e)}
    if multi and not a.no_port_peak and pair is not None:
        port_peak = {"pair_gbs": pair, "fanout_egress_gbs": fan,
                     "bytes_per_destination": 64 << 20,
                     "how": "ccube_measure_peer_bandwidth: 128-bit loads from local HBM, "
                            "128-bit stores into peer HBM, device-timed after ccube_barrier, "
                            "best of 5; fan-out m = every rank stores to m peers at once"}

    # ---- roofline of the (single) kernel
    hbm_peak, peak_src = measured_peaks()
    if not multi:
        alg_bytes = 2 * P * nbytes   # each rank's buffer read once + written once
        achieved = alg_bytes / (ms_step / 1e3) / 1e9
        roof = {"bound": "hbm", "achieved": achieved, "peak": hbm_peak, "unit": "GB/s",
                "frac": achieved / hbm_peak, "traffic": _ncu_traffic(a),
                "peak_source": peak_src,
                "algorithmic_bytes_per_launch": alg_bytes}
    else:
        roof = _nvlink_roofline(P, a.tree, nbytes, ms_step, port_peak)

    cpu = None
    oracle_check = None
    if rank == 0 and not a.no_cpu_baseline:
        nch = a.cpu_sample_chunks or 128
        if not multi:
            dt, sb, reps, want = oracle_time(P, a.tree, a.dtype, a.workload, a.chunk_bytes, nch,
                                             a.overlap, min_seconds=a.cpu_seconds)
            cbw, _ = busbw(sb, dt, P)
            cpu = {"value": cbw, "unit": "GB/s", "cores": 1, "kind": "oracle",
                   "sample": f"oracle.allreduce.replay on the first {nch} chunks ({sb} B per "
                             f"rank) of the {a.workload} gradient set, P={P}, {a.tree} tree, "
                             f"{'C1' if a.overlap else 'B'}; {reps} replays, {dt * reps:.1f} s "
                             f"of CPU work ({dt:.3f} s per replay)"}
            if a.cpu_cores != 1:
                xs_full = [h.view(torch.int16).numpy().view(np.uint16)
                           if a.dtype == "bfloat16" else h.numpy() for h in host] \
                    if not a.max_elems else None
                cpu["all_cores"] = oracle_time_parallel(P, a.tree, a.dtype, a.workload,
                                                        a.chunk_bytes, 32, a.overlap,
                                                        a.cpu_cores, a.cpu_seconds,
                                                        xs_full=xs_full)
            cpu["nproc"] = len(os.sched_getaffinity(0))
            cpu["cpu_model"] = _cpu_model()
        else:   # check only (no timing claim at N>1): the sample's oracle result
            _, _, _, want = oracle_time(P, a.tree, a.dtype, a.workload, a.chunk_bytes,
                                        min(nch, 8), a.overlap, max_reps=1)
        n = min(want.size, result_prefix.numel())   # --max-elems may cut the sample
        got = result_prefix[:n]
        got = got.view(torch.int16).numpy().view(np.uint16) if a.dtype == "bfloat16" \
            else got.numpy()
        oracle_check = {"elements": int(n), "source": "the cpu_baseline sample's oracle result",
                        "bitwise_equal": bool(np.array_equal(got, want[:n]))}

    # ---- NCCL on the same box and buffer (the comparison baseline, N>1 only)
    nccl = None
    if multi and not a.no_nccl and not shared:
        nccl = nccl_compare(a, dev, bufs[0], pristine[0], nbytes, P, stream)

    info = ccube.get_info()
    ccube.finalize()

    # ---- the other tree kinds and configs[2] (VGG-16 bf16, double tree) on this box:
    # the north-star target's double/rotated trees at >= 64 MB, next to configs[1]
    extra = None
    if not a.no_extra:
        extra = {}
        for kind in [k for k in ("single", "double", "rotated") if k != a.tree]:
            try:
                init(kind)
                try:
                    ms_k, tot_k = _time_steps(lambda: allreduce(bufs), restorer(bufs, pristine),
                                              a.extra_steps, 3, stream, multi, hdev)
                    ok_k, _ = _ranks_identical(bufs, multi, None if shared else dev)
                    extra[kind] = _extra_line(P, kind, nbytes, tot_k / a.extra_steps, multi,
                                              port_peak, ccube.get_info(), ok_k, a.workload,
                                              a.dtype)
                finally:
                    ccube.finalize()
            except Exception as e:  # noqa: BLE001 — reported; the main line stands
                extra[kind] = {"error": repr(e)}
        del bufs, pristine
        torch.cuda.empty_cache()
        if not a.max_elems:
            vcount = workloads.layer_ends("vgg16")[-1]
            g = torch.Generator(device=dev).manual_seed(20230225 + rank)
            vp = [torch.randn(vcount, device=dev, generator=g).to(torch.bfloat16)
                  for _ in my_ranks]
            vb = [p.clone() for p in vp]
            try:
                init("double")
                try:
                    ms_v, tot_v = _time_steps(lambda: allreduce(vb), restorer(vb, vp),
                                              a.extra_steps, 3, stream, multi, hdev)
                    ok_v, _ = _ranks_identical(vb, multi, None if shared else dev)
                    extra["vgg16_bf16_double"] = _extra_line(
                        P, "double", vcount * 2, tot_v / a.extra_steps, multi, port_peak,
                        ccube.get_info(), ok_v, "vgg16", "bfloat16")
                finally:
                    ccube.finalize()
            except Exception as e:  # noqa: BLE001 — reported; the main line stands
                extra["vgg16_bf16_double"] = {"error": repr(e)}
            if multi and not a.no_nccl and not shared:
                extra["vgg16_bf16_double"]["nccl"] = nccl_compare(a, dev, vb[0], vp[0],
                                                                  vcount * 2, P, stream)
            del vb, vp
    else:
        del bufs, pristine
    torch.cuda.empty_cache()

    iteration = None
    if not a.no_iter:
        try:
            iteration = run_iteration(a, P, log=_log, multi=multi, dev=dev, hdev=hdev)
        except Exception as e:  # noqa: BLE001 — reported in the line, the busbw stands
            iteration = {"error": repr(e)}

    if rank == 0:
        line = {
            "metric": METRIC, "value": bw, "unit": "GB/s", "n_gpus": world,
            "steps": a.steps, "warmup": a.warmup, "ms_per_step": ms_step,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": _dt(a.dtype), "data": "synthetic",
            "config": dict(_config(a, P, nbytes), channels=info["last_channels"],
                           ctas=info["last_ctas"], threads=info["last_threads"],
                           datapath="tma" if info["last_tma"] else "lsu",
                           l2=("inputs (P x bytes_per_rank) larger than L2 and restored from a "
                               "pristine copy between timed steps (flushes L2)") if not multi
                           else ("restored from a pristine copy between timed steps; per GPU "
                                 "the buffer (and the restore) is smaller than L2, so the "
                                 "kernel may start with L2-resident inputs")),
            "algbw": alg,
            "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "clocks": clk,
            "gpu_launches": a.steps * (2 if multi else 1),
            "ranks_identical": ok,
            "ms_per_step_p10_p50_p90": [float(np.percentile(ms, q)) for q in (10, 50, 90)],
            "ms_per_step_max": float(np.max(ms)),
            "iteration": iteration,
        }
        if multi:
            line["busbw_frac_of_900"] = bw / NVLINK_NOMINAL_GBS
            line["nvlink_counters_rank0"] = nvlink
            line["result_checksums"] = hashes
            line["port_peak"] = port_peak
        if oracle_check is not None:
            line["oracle_check"] = oracle_check
        if extra is not None:
            line["extra"] = extra
        if nccl is not None:
            line["nccl"] = nccl
        if placement_info is not None:
            line["placement"] = placement_info
        print(json.dumps(line), flush=True)
    if multi:
        dist.destroy_process_group()


def _nvlink_roofline(P, kind, nbytes, ms_step, port_peak):
    """N>1: the busiest port's bytes per direction (the method's algorithmic traffic,
    SURVEY §8(d)) over the kernel time, against the measured port peak."""
    port = max(_port_loads(P, kind)) * nbytes
    achieved = port / (ms_step / 1e3) / 1e9
    if port_peak is not None and "fanout_egress_gbs" in port_peak:
        peak = max(port_peak["fanout_egress_gbs"][1:])
        src = "measured: ccube_measure_peer_bandwidth, best fan-out egress per GPU"
    else:
        peak, src = NVLINK_MEASURED_GBS, "B200_PROFILING.md measured peer copy per direction"
    ceiling = _busbw_ceiling(P, kind)
    return {"bound": "nvlink", "achieved": achieved, "peak": peak, "unit": "GB/s",
            "frac": achieved / peak, "traffic": None, "peak_source": src,
            "frac_of_900": achieved / NVLINK_NOMINAL_GBS,
            "busbw_shape_ceiling_frac": ceiling,
            "algorithmic_bytes_per_launch": port}


def _busbw_ceiling(P, kind):
    """busbw ceiling as a fraction of the port rate for this tree shape: the ring's
    2(P-1)/P N per port over the busiest port's load."""
    return (2 * (P - 1) / P) / max(_port_loads(P, kind))


def _extra_line(P, kind, nbytes, ms, multi, port_peak, info, ok, workload, dtype):
    bw, alg = busbw(nbytes, ms / 1e3, P)
    d = {"workload": workload, "dtype": _dt(dtype), "tree": kind, "bytes_per_rank": nbytes,
         "ms_per_step": ms, "busbw": bw, "algbw": alg, "channels": info["last_channels"],
         "ctas": info["last_ctas"], "ranks_identical": ok}
    if multi:
        d["busbw_frac_of_900"] = bw / NVLINK_NOMINAL_GBS
        d["roofline"] = _nvlink_roofline(P, kind, nbytes, ms, port_peak)
    else:
        hbm, _ = measured_peaks()
        d["roofline"] = {"bound": "hbm", "achieved": 2 * P * nbytes / (ms / 1e3) / 1e9,
                         "peak": hbm, "frac": 2 * P * nbytes / (ms / 1e3) / 1e9 / hbm}
    return d


# ------------------------------------------------------- chained training iteration
ITER_MODES = ("compute", "B", "C1", "C2", "CC")   # paper's B / C1 / C2 / CC


def run_iteration(a, P, log=None, multi=False, dev=None, hdev=None):
    """Gradient-queue chaining (BASELINE.json configs[3]): synthetic ResNet-50 (or
    --iter-model) data-parallel iterations.

    One process per GPU (multi): one real model replica per GPU, its flat gradient
    queue reduced across the GPUs by the tree; iteration times are device-timed and
    the max over ranks.  Loopback (N=1): P logical ranks on one GPU, one model replica
    on local rank ``a.iter_rank``; the other ranks' backward output is emulated by a
    copy of the replica's gradients, inside the compute phase, and the AllReduce is
    limited to ``--iter-channels`` so the compute has SMs to overlap on.

    Modes: compute (no AllReduce), B (non-overlapped tree, unchained), C1
    (overlapped tree, unchained), C2 (B + per-layer gates), CC (C1 + gates), and with
    several GPUs R (NCCL ring AllReduce of the same buffer, unchained).  Unchained: the
    next forward waits for the whole AllReduce.  Chained: each layer's update+forward
    waits on its own gate (ccube_gradq_wait).  Returns {mode: ms/iteration},
    exposed = T_mode - T_compute, and the paper's normalized throughput
    throughput_P / (P * throughput_1GPU) = T_compute / T_mode (the compute-only
    iteration is the one-GPU iteration: same per-GPU batch, no communication)."""
    import torch
    import torch.distributed as dist
    import torch.nn.functional as F
    import torchvision
    from paper_conf_hpca_sanghoonsk23_b200 import ccube
    from paper_conf_hpca_sanghoonsk23_b200.gradient_queue import attach_gradient_queue

    dev = dev or torch.device("cuda", torch.cuda.current_device())
    torch.manual_seed(0)
    torch.backends.cudnn.benchmark = True
    model = _iter_model(a.iter_model).to(dev).to(memory_format=torch.channels_last)
    rr = None if multi else a.iter_rank % P
    gq = attach_gradient_queue(model, lr=1e-3, world_size=P, local_rank=rr,
                               fused_sgd=a.iter_fused_sgd)
    gq.update = True
    B = a.iter_batch
    x = torch.randn(B, 3, 224, 224, device=dev).to(memory_format=torch.channels_last)
    y = torch.randint(0, 1000, (B,), device=dev)
    others = [] if multi else [torch.zeros_like(gq.flat) for _ in range(P - 1)]
    bufs = [gq.flat] if multi else others[:rr] + [gq.flat] + others[rr:]
    wts = None
    if a.iter_fused_sgd and not multi:   # the emulated replicas' weights, updated too
        ow = [gq.flat_w.clone() for _ in range(P - 1)]
        wts = ow[:rr] + [gq.flat_w] + ow[rr:]
    comp, comm = torch.cuda.Stream(), torch.cuda.Stream()
    modes = ITER_MODES + (("R",) if multi and dev is not None and hdev is not None else ())
    ring = None
    if "R" in modes:
        saved = os.environ.get("NCCL_ALGO")
        os.environ["NCCL_ALGO"] = "Ring"
        ring = dist.new_group(backend="nccl")
        if saved is None:
            os.environ.pop("NCCL_ALGO", None)
        else:
            os.environ["NCCL_ALGO"] = saved
    if multi:
        ccube.init_distributed(dist.group.WORLD, tree=a.iter_tree, chunk_bytes=a.chunk_bytes)
    else:
        ccube.init_loopback(P, a.iter_tree, a.chunk_bytes)
    res = {}
    try:
        channels = a.iter_channels if not multi else a.iter_channels_multi
        ccube.set_channels(channels)
        gq.set_layers(weights=wts)

        ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731

        def allreduce():
            if multi:
                ccube.allreduce_tree(gq.flat, stream=comm)
            else:
                ccube.allreduce_tree_local(bufs, stream=comm)

        def one(mode, marks=None):
            with torch.cuda.stream(comp):
                with torch.autocast("cuda", dtype=torch.bfloat16):
                    out = model(x)
                    loss = F.cross_entropy(out.float(), y)
                if marks is not None:
                    marks["fwd_end"] = ev()
                    marks["fwd_end"].record(comp)
                comp.wait_stream(comm)    # the AllReduce is done reading/writing the queue
                gq.zero_()
                loss.backward()
                for o in others:          # emulated replicas' backward output (loopback)
                    o.copy_(gq.flat)
            if mode != "compute":
                comm.wait_stream(comp)
                if marks is not None:
                    marks["ar0"] = ev()
                    marks["ar0"].record(comm)
                if mode == "R":
                    with torch.cuda.stream(comm):
                        dist.all_reduce(gq.flat, group=ring)
                else:
                    allreduce()
                if marks is not None:
                    marks["ar1"] = ev()
                    marks["ar1"].record(comm)
                if mode in ("B", "C1", "R"):
                    comp.wait_stream(comm)

        runs = {m: [] for m in modes}
        timeline = {}
        for rnd in range(a.iter_rounds):          # modes interleaved, median over rounds
            for mode in modes:
                ccube.set_overlap(mode in ("C1", "CC"))
                gq.chained = mode in ("C2", "CC")
                # compute-only and R have no C-Cube AllReduce to ride on: hooks update
                gq.fused_sgd = a.iter_fused_sgd and mode not in ("compute", "R")
                for _ in range(a.iter_warmup):
                    one(mode)
                torch.cuda.synchronize()
                if multi:
                    dist.barrier()
                e0, e1 = ev(), ev()
                e0.record(comp)
                for _ in range(a.iter_steps):
                    one(mode)
                comp.wait_stream(comm)
                e1.record(comp)
                if rnd == 0:   # one instrumented pair: AllReduce of i, forward of i+1
                    m0, m1 = {}, {}
                    one(mode, m0)
                    one(mode, m1)
                    comp.wait_stream(comm)
                torch.cuda.synchronize()
                t = e0.elapsed_time(e1) / a.iter_steps
                if multi:
                    t = _allmax(t, hdev)
                runs[mode].append(t)
                if rnd == 0:
                    tl = {"forward_end_after_allreduce_end_ms": None}
                    if mode != "compute":
                        tl["allreduce_ms"] = m0["ar0"].elapsed_time(m0["ar1"])
                        tl["forward_end_after_allreduce_end_ms"] = \
                            m0["ar1"].elapsed_time(m1["fwd_end"])
                    timeline[mode] = tl
                gq.chained = False
                if log and (not multi or dist.get_rank() == 0):
                    log(f"[iter] round {rnd} {mode}: {runs[mode][-1]:.3f} ms/iter")
        res = {m: float(np.median(v)) for m, v in runs.items()}
    finally:
        gq.remove()
        ccube.finalize()
        if ring is not None:
            dist.destroy_process_group(ring)
    t0 = res["compute"]
    out = {"unit": "ms/iter", "batch_per_gpu": B, "P": P, "tree": a.iter_tree,
           "channels": channels, "fused_sgd": a.iter_fused_sgd,
           "model": f"{a.iter_model} (random init), bf16 autocast, channels_last",
           "grad_bytes_per_rank": gq.numel * 4,
           "ms": res, "exposed_ms": {m: res[m] - t0 for m in modes if m != "compute"},
           "normalized_throughput": {m: t0 / res[m] for m in modes if m != "compute"},
           "runs_ms": runs, "timeline": timeline, "rounds": a.iter_rounds,
           "steps_per_round": a.iter_steps}
    if multi:
        out["note"] = ("one model replica per GPU; device time per iteration, max over ranks; "
                       "R = NCCL_ALGO=Ring all_reduce of the same flat buffer")
    else:
        out["replica_rank"] = rr
        out["note"] = "loopback: P logical ranks share one GPU's SMs and HBM with the compute"
    exp = out["exposed_ms"]
    cut = lambda m, ref: (1 - exp[m] / exp[ref]) if exp[ref] > 0 else None  # noqa: E731
    out["exposed_cut_CC_vs_B"] = cut("CC", "B")
    out["exposed_cut_C2_vs_B"] = cut("C2", "B")      # chaining alone
    out["exposed_cut_CC_vs_C1"] = cut("CC", "C1")    # chaining on top of the overlapped tree
    if "R" in exp:
        out["exposed_cut_CC_vs_R"] = cut("CC", "R")
    return out


def _iter_model(name):
    """torchvision ResNet-50 / VGG-16, or the ZFNet-like net of workloads.py."""
    import torchvision
    if name == "zfnet":
        from paper_conf_hpca_sanghoonsk23_b200.workloads import zfnet
        return zfnet()
    return getattr(torchvision.models, name)(weights=None)


def _allmax(x, dev):
    """Max over ranks of a host float (on ``dev`` for NCCL, on the host for gloo)."""
    import torch
    import torch.distributed as dist
    t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return t.item()


def nccl_compare(a, dev, buf, pristine, nbytes, P, stream):
    """NCCL AllReduce (sum) on the same buffer, dtype and timing protocol as the
    C-Cube arm: Ring, Tree and NCCL's own default choice.  NCCL_ALGO is read when a
    communicator is created, so each algorithm gets a fresh group created after the
    variable is set.  Returns {algo: {"busbw": GB/s, "ms_per_step": ms}}."""
    import torch
    import torch.distributed as dist

    out = {}
    saved = os.environ.get("NCCL_ALGO")
    for algo in ("Ring", "Tree", "default"):
        if algo == "default":
            os.environ.pop("NCCL_ALGO", None)
        else:
            os.environ["NCCL_ALGO"] = algo
        try:
            g = dist.new_group(backend="nccl")
            with torch.cuda.stream(stream):
                for _ in range(max(3, a.warmup)):
                    buf.copy_(pristine)
                    dist.all_reduce(buf, group=g)
            torch.cuda.synchronize()
            evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                   for _ in range(a.nccl_steps)]
            dist.barrier()
            torch.cuda.synchronize()
            with torch.cuda.stream(stream):
                for s, e in evs:
                    buf.copy_(pristine)
                    s.record(stream)
                    dist.all_reduce(buf, group=g)
                    e.record(stream)
            torch.cuda.synchronize()
            t = torch.tensor([sum(s.elapsed_time(e) for s, e in evs)], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = t.item() / a.nccl_steps
            bw, alg = busbw(nbytes, ms / 1e3, P)
            out[algo] = {"busbw": bw, "algbw": alg, "ms_per_step": ms,
                         "busbw_frac_of_900": bw / NVLINK_NOMINAL_GBS}
            dist.destroy_process_group(g)
        except Exception as e:  # noqa: BLE001 — reported in the line, the C-Cube arm stands
            out[algo] = {"error": repr(e)}
    if saved is None:
        os.environ.pop("NCCL_ALGO", None)
    else:
        os.environ["NCCL_ALGO"] = saved
    return out


def _port_loads(P, kind):
    """Bytes each rank sends per direction per byte of buffer (library trees)."""
    from paper_conf_hpca_sanghoonsk23_b200 import ccube
    ntrees = {"single": 1, "double": 2, "rotated": P if P > 1 else 1}[kind]
    loads = [0.0] * P
    for t in range(ntrees):
        par = ccube.tree_parents(P, kind, t)
        for v in range(P):
            nchild = sum(1 for u in range(P) if par[u] == v)
            loads[v] += (nchild + (1 if par[v] >= 0 else 0)) / ntrees
    return loads


def _ncu_traffic(a):
    """dram bytes per launch from the committed ncu --set full capture, if it was
    taken on this line's configuration (the default bench workload), else None."""
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(path) as f:
            d = json.load(f)
    except Exception:  # noqa: BLE001
        return None
    cfg = d.get("config", {})
    mine = {"workload": a.workload, "tree": a.tree, "ranks": a.ranks, "dtype": a.dtype,
            "chunk_bytes": a.chunk_bytes, "overlap": a.overlap}
    return d.get("dram_bytes_per_launch") if cfg == mine else None


def _log(msg):
    print(msg, file=sys.stderr, flush=True)


def run_iter_only(a):
    """--mode iter: only the chained-vs-unchained iteration (loopback, N=1)."""
    import torch
    torch.cuda.set_device(0)
    it = run_iteration(a, a.ranks, log=_log)
    line = {"metric": f"iter time chained vs unchained (synthetic {a.iter_model} DP iteration)",
            "value": it["ms"]["CC"], "unit": "ms/iter", "n_gpus": 1,
            "steps": a.iter_steps, "warmup": a.iter_warmup, "higher_is_better": False,
            "dtype": "bf16 compute / f32 gradients", "data": "synthetic",
            "config": {"workload": f"{a.iter_model} iteration, batch {a.iter_batch}, P={a.ranks} "
                                   f"logical ranks (loopback), {a.iter_tree} tree"},
            "iteration": it}
    print(json.dumps(line), flush=True)


def main():
    a = parse()
    if a.impl == "reference":
        run_reference(a)
    elif a.mode == "iter":
        run_iter_only(a)
    else:
        run_ccube(a)


if __name__ == "__main__":
    main()

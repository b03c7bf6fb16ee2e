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


def parse():
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
    p.add_argument("--iter-model", choices=["resnet50", "vgg16"], default="resnet50")
    p.add_argument("--iter-fused-sgd", action="store_true",
                   help="apply the SGD step inside the AllReduce kernel (f2)")
    p.add_argument("--iter-steps", type=int, default=20)
    p.add_argument("--iter-rounds", type=int, default=5)
    p.add_argument("--iter-warmup", type=int, default=2)
    p.add_argument("--iter-channels", type=int, default=4)
    p.add_argument("--iter-tree", choices=["single", "double", "rotated"], default="single")
    p.add_argument("--iter-rank", type=int, default=1,
                   help="loopback rank that hosts the model replica (1 = a leaf of tree 0)")
    a = p.parse_args()
    if a.dtype is None:
        a.dtype = "bfloat16" if a.workload == "vgg16" else "float32"
    if a.tree is None:
        a.tree = "double" if a.workload == "vgg16" else "single"
    return a


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
    """Seconds for one run of the CPU oracle's message-passing replay on ``xs``."""
    from oracle import allreduce as oar
    t0 = time.perf_counter()
    oar.replay(xs, tree, chunk_bytes, dtype, overlap=bool(overlap))
    return time.perf_counter() - t0


def oracle_time(P, tree, dtype, workload, chunk_bytes, nchunks, overlap, min_seconds=0.0,
                max_reps=64):
    """Time the CPU oracle's replay on the first ``nchunks`` chunks of the workload
    (every rank's data for those chunks), repeated until at least ``min_seconds`` of
    CPU work (at most ``max_reps`` replays).  Returns (seconds per replay, bytes per
    rank per replay, replays)."""
    xs, nbytes = oracle_inputs(P, dtype, workload, chunk_bytes, nchunks)
    reps, total = 0, 0.0
    while reps == 0 or (total < min_seconds and reps < max_reps):
        total += oracle_replay_time(xs, tree, dtype, chunk_bytes, overlap)
        reps += 1
    return total / reps, nbytes, reps


def busbw(bytes_per_rank, seconds, P):
    alg = bytes_per_rank / seconds / 1e9
    return alg * 2 * (P - 1) / P, alg


def run_reference(a):
    """--impl reference: the CPU oracle as it stands, on the host cores (rank 0 only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    P = a.ranks if a.gpus == 1 else a.gpus
    nchunks = a.cpu_sample_chunks or 128  # 128 chunks x 256 KiB = 32 MiB per rank (of 102 MB)
    xs, nbytes = oracle_inputs(P, a.dtype, a.workload, a.chunk_bytes, nchunks)
    for _ in range(a.warmup):
        oracle_replay_time(xs, a.tree, a.dtype, a.chunk_bytes, a.overlap)
    total = 0.0
    for _ in range(a.steps):
        total += oracle_replay_time(xs, a.tree, a.dtype, a.chunk_bytes, a.overlap)
    bw, alg = busbw(nbytes, total / a.steps, P)
    sample = (f"oracle.allreduce.replay on the first {nchunks} chunks ({nbytes} B per rank) of the "
              f"{a.workload} gradient set, P={P}, {a.tree} tree, one step = one replay")
    line = {
        "impl": "reference", "metric": METRIC, "value": bw, "unit": "GB/s", "n_gpus": a.gpus,
        "steps": a.steps, "warmup": a.warmup, "ms_per_step": total / a.steps * 1e3,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": _dt(a.dtype),
        "data": "synthetic", "config": _config(a, P, nbytes),
        "cpu_baseline": {"value": bw, "unit": "GB/s", "cores": 1, "kind": "oracle",
                         "sample": sample},
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
    if multi:
        ccube.init_distributed(dist.group.WORLD, tree=a.tree, chunk_bytes=a.chunk_bytes)
    else:
        ccube.init_loopback(P, a.tree, a.chunk_bytes)
    if a.channels:
        ccube.set_channels(a.channels)
    if a.threads:
        ccube.set_threads(a.threads)
    if a.datapath:
        ccube.set_datapath(a.datapath)
    ccube.set_overlap(bool(a.overlap))
    stream = torch.cuda.Stream()

    def step():
        if multi:
            ccube.allreduce_tree(bufs[0], stream=stream)
        else:
            ccube.allreduce_tree_local(bufs, stream=stream)

    def restore():
        with torch.cuda.stream(stream):
            for b, p in zip(bufs, pristine):
                b.copy_(p)   # > L2 (126 MB): also flushes L2 between timed iterations

    # warm-up
    for _ in range(max(3, a.warmup)):
        restore()
        step()
    torch.cuda.synchronize()
    clocks = ClockSampler(local_rank if multi else 0, enabled=(rank == 0 and not a.no_clocks))
    time.sleep(0.3)
    # timed region: K steps, each bracketed by events on the launching stream
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
           for _ in range(a.steps)]
    if multi:
        dist.barrier()
    torch.cuda.synchronize()
    for i in range(a.steps):
        restore()
        evs[i][0].record(stream)
        step()
        evs[i][1].record(stream)
    torch.cuda.synchronize()
    if multi:
        dist.barrier()
    ms = [s.elapsed_time(e) for s, e in evs]
    total_ms = float(np.sum(ms))
    if multi:
        total_ms = _allmax(total_ms, None if shared else dev)
    clk = clocks.stop()
    ms_step = total_ms / a.steps
    bw, alg = busbw(nbytes, ms_step / 1e3, P)

    # correctness spot-check of the timed configuration (all ranks identical)
    ok = True
    if not multi:
        ok = all(torch.equal(bufs[r], bufs[0]) for r in range(1, P))

    # ---- e2e: host buffers -> device -> allreduce -> host, through the public API.
    # Every step copies its inputs in from pinned host memory and its results out.
    # Two device buffer sets alternate so that step i's device->host copy (second
    # stream, the other copy engine) overlaps step i+1's host->device copy.
    e2e = None
    if not a.no_e2e:
        outs = [torch.empty_like(h).pin_memory() for h in host]
        sets = [bufs, [torch.empty_like(b) for b in bufs]]
        dstream = torch.cuda.Stream()
        ev = lambda: torch.cuda.Event()  # noqa: E731
        d2h_done = [None, None]

        def e2e_step(i):
            s_ = i % 2
            if d2h_done[s_] is not None:          # step i-2's results are out of this set
                stream.wait_event(d2h_done[s_])
            with torch.cuda.stream(stream):
                for b, h in zip(sets[s_], host):
                    b.copy_(h, non_blocking=True)
            if multi:
                ccube.allreduce_tree(sets[s_][0], stream=stream)
            else:
                ccube.allreduce_tree_local(sets[s_], stream=stream)
            k = ev()
            k.record(stream)
            dstream.wait_event(k)
            with torch.cuda.stream(dstream):
                for o, b in zip(outs, sets[s_]):
                    o.copy_(b, non_blocking=True)
            d2h_done[s_] = ev()
            d2h_done[s_].record(dstream)

        for i in range(2):
            e2e_step(i)
        torch.cuda.synchronize()
        if multi:
            dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for i in range(a.e2e_steps):
            e2e_step(i)
        stream.wait_stream(dstream)
        e1.record(stream)
        torch.cuda.synchronize()
        e2e_ms = e0.elapsed_time(e1) / a.e2e_steps
        if multi:
            e2e_ms = _allmax(e2e_ms, None if shared else dev)
        ebw, _ = busbw(nbytes, e2e_ms / 1e3, P)
        ok_e2e = all(torch.equal(o, outs[0]) for o in outs[1:]) if not multi else None
        e2e = {"value": ebw, "unit": "GB/s", "ms_per_step": e2e_ms,
               "h2d_bytes_per_step": nbytes * len(my_ranks),
               "d2h_bytes_per_step": nbytes * len(my_ranks), "steps": a.e2e_steps,
               "pipelining": "two device buffer sets; step i's D2H overlaps step i+1's H2D",
               "ranks_identical": ok_e2e}
        del sets

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
        port = max(_port_loads(P, a.tree)) * nbytes
        achieved = port / (ms_step / 1e3) / 1e9
        roof = {"bound": "nvlink", "achieved": achieved, "peak": NVLINK_MEASURED_GBS,
                "unit": "GB/s", "frac": achieved / NVLINK_MEASURED_GBS, "traffic": None,
                "peak_source": "B200_PROFILING.md measured peer copy per direction",
                "algorithmic_bytes_per_launch": port}

    cpu = None
    if rank == 0 and not a.no_cpu_baseline:
        nch = a.cpu_sample_chunks or 128
        dt, sb, reps = oracle_time(P, a.tree, a.dtype, a.workload, a.chunk_bytes, nch, a.overlap,
                                   min_seconds=a.cpu_seconds)
        cbw, _ = busbw(sb, dt, P)
        cpu = {"value": cbw, "unit": "GB/s", "cores": 1, "kind": "oracle",
               "sample": f"oracle.allreduce.replay on the first {nch} chunks ({sb} B per rank) "
                         f"of the {a.workload} gradient set, P={P}, {a.tree} tree, "
                         f"{'C1' if a.overlap else 'B'}; {reps} replays, {dt * reps:.1f} s of "
                         f"CPU work ({dt:.3f} s per replay)"}

    # ---- NCCL on the same box and buffer (the comparison baseline, N>1 only)
    nccl = None
    if multi and not a.no_nccl and not shared:
        nccl = nccl_compare(a, dev, bufs[0], pristine[0], nbytes, P, stream)

    info = ccube.get_info()
    ccube.finalize()
    iteration = None
    if not multi and not a.no_iter:
        del bufs, pristine
        torch.cuda.empty_cache()
        try:
            iteration = run_iteration(a, P, log=_log)
        except Exception as e:  # noqa: BLE001 — reported in the line, the busbw stands
            iteration = {"error": repr(e)}

    if rank == 0:
        line = {
            "metric": METRIC, "value": bw, "unit": "GB/s", "n_gpus": world,
            "steps": a.steps, "warmup": a.warmup, "ms_per_step": ms_step,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": _dt(a.dtype), "data": "synthetic",
            "config": dict(_config(a, P, nbytes), channels=info["last_channels"],
                           ctas=info["last_ctas"], threads=info["threads"],
                           datapath="tma" if info["last_tma"] else "lsu",
                           l2="inputs (P x bytes_per_rank) larger than L2 and restored from a "
                              "pristine copy between timed steps (flushes L2)"),
            "algbw": alg, "busbw_frac_of_900": bw / NVLINK_NOMINAL_GBS,
            "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "clocks": clk,
            "gpu_launches": a.steps, "ranks_identical": ok,
            "ms_per_step_p10_p50_p90": [float(np.percentile(ms, q)) for q in (10, 50, 90)],
            "iteration": iteration,
        }
        if nccl is not None:
            line["nccl"] = nccl
        if placement_info is not None:
            line["placement"] = placement_info
        print(json.dumps(line), flush=True)
    if multi:
        dist.destroy_process_group()


# ------------------------------------------------------- chained training iteration
ITER_MODES = ("compute", "B", "C1", "C2", "CC")   # paper's B / C1 / C2 / CC


def run_iteration(a, P, log=None):
    """Gradient-queue chaining (BASELINE.json configs[3]): synthetic ResNet-50
    data-parallel iterations, loopback (P logical ranks on one GPU, one model
    replica on local rank ``a.iter_rank``; the other ranks' backward output is
    emulated by a copy of the replica's gradients, inside the compute phase).

    Modes: compute (no AllReduce), B (non-overlapped tree, unchained), C1
    (overlapped tree, unchained), C2 (B + per-layer gates), CC (C1 + gates).
    Unchained: the next forward waits for the whole AllReduce.  Chained: each
    layer's update+forward waits on its own gate (ccube_gradq_wait).
    Returns {mode: ms per iteration} and exposed = T_mode - T_compute."""
    import torch
    import torch.nn.functional as F
    import torchvision
    from paper_conf_hpca_sanghoonsk23_b200 import ccube
    from paper_conf_hpca_sanghoonsk23_b200.gradient_queue import attach_gradient_queue

    dev = torch.device("cuda", torch.cuda.current_device())
    torch.manual_seed(0)
    torch.backends.cudnn.benchmark = True
    model = getattr(torchvision.models, a.iter_model)(weights=None)
    model = model.to(dev).to(memory_format=torch.channels_last)
    rr = a.iter_rank % P
    gq = attach_gradient_queue(model, lr=1e-3, world_size=P, local_rank=rr,
                               fused_sgd=a.iter_fused_sgd)
    gq.update = True
    B = a.iter_batch
    x = torch.randn(B, 3, 224, 224, device=dev).to(memory_format=torch.channels_last)
    y = torch.randint(0, 1000, (B,), device=dev)
    others = [torch.zeros_like(gq.flat) for _ in range(P - 1)]
    bufs = others[:rr] + [gq.flat] + others[rr:]
    wts = None
    if a.iter_fused_sgd:   # the emulated replicas' weights, updated by the kernel too
        ow = [gq.flat_w.clone() for _ in range(P - 1)]
        wts = ow[:rr] + [gq.flat_w] + ow[rr:]
    comp, comm = torch.cuda.Stream(), torch.cuda.Stream()
    ccube.init_loopback(P, a.iter_tree, a.chunk_bytes)
    res = {}
    try:
        ccube.set_channels(a.iter_channels)
        gq.set_layers(weights=wts)

        ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731

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
                for o in others:          # emulated replicas' backward output
                    o.copy_(gq.flat)
            if mode != "compute":
                comm.wait_stream(comp)
                if marks is not None:
                    marks["ar0"] = ev()
                    marks["ar0"].record(comm)
                ccube.allreduce_tree_local(bufs, stream=comm)
                if marks is not None:
                    marks["ar1"] = ev()
                    marks["ar1"].record(comm)
                if mode in ("B", "C1"):
                    comp.wait_stream(comm)

        runs = {m: [] for m in ITER_MODES}
        timeline = {}
        for rnd in range(a.iter_rounds):          # modes interleaved, median over rounds
            for mode in ITER_MODES:
                ccube.set_overlap(mode in ("C1", "CC"))
                gq.chained = mode in ("C2", "CC")
                # compute-only has no AllReduce to ride on: the hooks update instead
                gq.fused_sgd = a.iter_fused_sgd and mode != "compute"
                for _ in range(a.iter_warmup):
                    one(mode)
                torch.cuda.synchronize()
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
                runs[mode].append(e0.elapsed_time(e1) / a.iter_steps)
                if rnd == 0:
                    tl = {"forward_end_after_allreduce_end_ms": None}
                    if mode != "compute":
                        tl["allreduce_ms"] = m0["ar0"].elapsed_time(m0["ar1"])
                        tl["forward_end_after_allreduce_end_ms"] = \
                            m0["ar1"].elapsed_time(m1["fwd_end"])
                    timeline[mode] = tl
                gq.chained = False
                if log:
                    log(f"[iter] round {rnd} {mode}: {runs[mode][-1]:.3f} ms/iter")
        res = {m: float(np.median(v)) for m, v in runs.items()}
    finally:
        gq.remove()
        ccube.finalize()
    t0 = res["compute"]
    out = {"unit": "ms/iter", "batch": B, "P": P, "tree": a.iter_tree,
           "channels": a.iter_channels, "replica_rank": rr,
           "fused_sgd": a.iter_fused_sgd,
           "model": f"torchvision {a.iter_model} (random init), bf16 autocast, channels_last",
           "grad_bytes_per_rank": gq.numel * 4,
           "ms": res, "exposed_ms": {m: res[m] - t0 for m in ITER_MODES if m != "compute"},
           "runs_ms": runs, "timeline": timeline, "rounds": a.iter_rounds,
           "steps_per_round": a.iter_steps,
           "note": "loopback: P logical ranks share one GPU's SMs and HBM with the compute"}
    exp = out["exposed_ms"]
    cut = lambda m, ref: (1 - exp[m] / exp[ref]) if exp[ref] > 0 else None  # noqa: E731
    out["exposed_cut_CC_vs_B"] = cut("CC", "B")
    out["exposed_cut_C2_vs_B"] = cut("C2", "B")      # chaining alone
    out["exposed_cut_CC_vs_C1"] = cut("CC", "C1")    # chaining on top of the overlapped tree
    return out


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

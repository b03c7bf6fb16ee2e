"""GPU parity: the CUDA path through the C ABI vs the CPU oracle (loopback mode:
P logical ranks on one B200, same kernel body as one-process-per-GPU).

Bar (north star / DESIGN.md §5): bit-exact for int32, fp32 and bf16 (same fixed
order and per-node rounding); every rank identical; B == C1 bitwise; normwise
error vs an fp64 sum <= 1e-6 (fp32) and <= 1e-2 (bf16)."""

import numpy as np
import pytest
import torch

from oracle import allreduce as oar
from oracle import arith, partition
from paper_conf_hpca_sanghoonsk23_b200 import ccube, inputs, workloads

from gpu_helpers import device_inputs, oracle_chunk, to_numpy, to_torch

pytestmark = pytest.mark.gpu


@pytest.fixture
def comm():
    """Yields an init function; always finalizes."""
    state = {"on": False}

    def _init(P, kind="single", chunk_bytes=4096, channels=None, overlap=True, threads=None,
              transport=None):
        ccube.init_loopback(P, kind, chunk_bytes)
        state["on"] = True
        if transport is not None:
            ccube.set_transport(transport)
        if channels is not None:
            ccube.set_channels(channels)
        if threads is not None:
            ccube.set_threads(threads)
        ccube.set_overlap(overlap)

    yield _init
    if state["on"]:
        ccube.finalize()


def _run(P, kind, dtype, count, chunk_bytes, seed=5):
    xs = [inputs.gradients(r, count, dtype, seed=seed) for r in range(P)]
    ts = [to_torch(x, dtype).cuda() for x in xs]
    ccube.allreduce_tree_local(ts)
    torch.cuda.synchronize()
    return xs, [to_numpy(t, dtype) for t in ts]


@pytest.mark.parametrize("P", [2, 3, 4, 5, 8])
@pytest.mark.parametrize("kind", ["single", "double"])
@pytest.mark.parametrize("dtype", ["int32", "float32", "bfloat16"])
@pytest.mark.parametrize("overlap", [True, False])
@pytest.mark.parametrize("transport", ["pull", "push"])
def test_parity_small(comm, P, kind, dtype, overlap, transport):
    """Several chunks (K = 8), 4 channels, ragged tail (not a whole vector); both edge
    transports (PUSH = the cross-GPU path, PULL = the same-GPU path)."""
    chunk = 4096
    comm(P, kind, chunk, channels=4, overlap=overlap, transport=transport)
    E = chunk // arith.ELEM_SIZE[dtype]
    count = 7 * E + 13
    xs, outs = _run(P, kind, dtype, count, chunk)
    ref = oar.reference(xs, kind, chunk, dtype)[0]
    for r in range(P):
        assert np.array_equal(outs[r], ref), f"rank {r}"


@pytest.mark.parametrize("channels", [0, 1, 2, 3, 5, 7, 8, 16])
def test_parity_channels(comm, channels):
    """Channel slices need not divide the chunk (0 = auto: as many as fit)."""
    chunk = 16 * 1024 * 3
    comm(8, "double", chunk, channels=channels, threads=256)
    count = 5 * chunk // 4 + 1001
    xs, outs = _run(8, "double", "float32", count, chunk)
    ref = oar.reference(xs, "double", chunk, "float32")[0]
    for r in range(8):
        assert np.array_equal(outs[r], ref)


@pytest.mark.parametrize("threads", [32, 64, 128, 256])
def test_parity_threads(comm, threads):
    comm(4, "single", 8192, channels=2, threads=threads)
    xs, outs = _run(4, "single", "bfloat16", 40000 + 3, 8192)
    ref = oar.reference(xs, "single", 8192, "bfloat16")[0]
    for r in range(4):
        assert np.array_equal(outs[r], ref)


def test_repeated_calls_advance_epochs(comm):
    comm(8, "double", 4096, channels=4)
    for it in range(6):
        if it == 3:
            ccube.set_transport("push")   # params rebuilt, counters keep advancing
        count = [5000, 20000, 7, 12345, 99, 40000][it]
        xs, outs = _run(8, "double", "float32", count, 4096, seed=100 + it)
        ref = oar.reference(xs, "double", 4096, "float32")[0]
        for r in range(8):
            assert np.array_equal(outs[r], ref), (it, r)
    info = ccube.get_info()
    assert info["epoch_base"][0] > 0 and info["epoch_base"][1] > 0


@pytest.mark.parametrize("count", [1, 3, 4, 5, 1023, 1024, 1025])
def test_tiny_and_boundary_counts(comm, count):
    comm(4, "double", 4096, channels=4)
    xs, outs = _run(4, "double", "float32", count, 4096)
    ref = oar.reference(xs, "double", 4096, "float32")[0]
    for r in range(4):
        assert np.array_equal(outs[r], ref)


def test_count_zero_and_P1_are_noops(comm):
    comm(4, "single", 4096, channels=4)
    ts = [torch.arange(100, dtype=torch.float32, device="cuda") + r for r in range(4)]
    keep = [t.clone() for t in ts]
    ccube.allreduce_tree_local(ts, count=0)
    torch.cuda.synchronize()
    for a, b in zip(ts, keep):
        assert torch.equal(a, b)


def test_P1_loopback_noop():
    ccube.init_loopback(1, "single", 4096)
    try:
        t = torch.arange(100, dtype=torch.float32, device="cuda")
        ccube.allreduce_tree_local([t])
        torch.cuda.synchronize()
        assert torch.equal(t, torch.arange(100, dtype=torch.float32, device="cuda"))
    finally:
        ccube.finalize()


def test_misaligned_buffer_rejected(comm):
    comm(2, "single", 4096, channels=4)
    base = [torch.zeros(1000, dtype=torch.float32, device="cuda") for _ in range(2)]
    with pytest.raises(ccube.CCubeError) as e:
        ccube.allreduce_tree_local([b[1:] for b in base])
    assert e.value.code == ccube.ERR_INVALID_ARG
    assert "aligned" in ccube.last_error()


def test_too_many_channels_rejected(comm):
    comm(8, "double", 1 << 20, channels=64)
    ts = [torch.zeros(1 << 20, device="cuda") for _ in range(8)]
    with pytest.raises(ccube.CCubeError) as e:
        ccube.allreduce_tree_local(ts)
    assert e.value.code == ccube.ERR_UNSUPPORTED


def test_int32_full_range_wraps(comm):
    comm(8, "single", 4096, channels=4)
    count = 9000
    xs = [inputs.gradients(r, count, "int32", seed=9, full_range=True) for r in range(8)]
    ts = [to_torch(x, "int32").cuda() for x in xs]
    ccube.allreduce_tree_local(ts)
    s = np.zeros(count, dtype=np.int64)
    for x in xs:
        s += x.astype(np.int64)
    want = ((s + 2 ** 31) % 2 ** 32 - 2 ** 31).astype(np.int32)
    for t in ts:
        assert np.array_equal(to_numpy(t, "int32"), want)


def _full_size(P, kind, dtype, workload, chunk_bytes, overlap=True):
    ends = workloads.layer_ends(workload)
    count = ends[-1]
    ts = device_inputs(P, count, dtype, layer_ends=ends)
    ccube.set_overlap(overlap)
    ccube.allreduce_tree_local(ts)
    torch.cuda.synchronize()
    return count, ends, ts


@pytest.mark.parametrize("kind", ["single", "double"])
@pytest.mark.parametrize("transport", ["auto", "push"])
def test_full_size_resnet50_fp32(comm, kind, transport):
    """configs[1]: ResNet-50 gradient set (25,557,032 fp32, K = 390) at P = 8 with the
    bench's launch configuration; sampled chunks bit-exact vs the oracle (first,
    last ragged, random), every rank identical, fp64 normwise error <= 1e-6."""
    P, chunk = 8, 256 << 10
    comm(P, kind, chunk, transport=transport)
    count, ends, ts = _full_size(P, kind, "float32", "resnet50", chunk)
    K = partition.num_chunks(count, chunk, 4)
    assert K == 390
    rng = np.random.default_rng(0)
    for c in sorted({0, 1, K - 2, K - 1, *rng.integers(0, K, 6).tolist()}):
        lo, hi, want = oracle_chunk(P, kind, chunk, "float32", count, c, layer_ends=ends)
        for r in (0, 3, 7):
            assert np.array_equal(to_numpy(ts[r][lo:hi], "float32"), want), (c, r)
    for r in range(1, P):
        assert torch.equal(ts[r], ts[0])
    # order-independent fp64 reference on the device (a check, not the product path)
    s = torch.zeros(count, dtype=torch.float64, device="cuda")
    for x in device_inputs(P, count, "float32", layer_ends=ends):
        s += x.double()
    err = (ts[0].double() - s).norm() / s.norm()
    assert err.item() <= 1e-6


def test_full_size_vgg16_bf16_double(comm):
    """configs[2]: VGG-16 bf16 gradients (138,357,544, K = 1056) on the double tree."""
    P, chunk = 8, 256 << 10
    comm(P, "double", chunk)
    count, ends, ts = _full_size(P, "double", "bfloat16", "vgg16", chunk)
    K = partition.num_chunks(count, chunk, 2)
    assert K == 1056
    for c in (0, 1, 500, 777, K - 2, K - 1):
        lo, hi, want = oracle_chunk(P, "double", chunk, "bfloat16", count, c, layer_ends=ends)
        for r in (0, 5):
            assert np.array_equal(to_numpy(ts[r][lo:hi], "bfloat16"), want), (c, r)
    for r in range(1, P):
        assert torch.equal(ts[r], ts[0])
    s = torch.zeros(count, dtype=torch.float64, device="cuda")
    for x in device_inputs(P, count, "bfloat16", layer_ends=ends):
        s += x.double()
    err = (ts[0].double() - s).norm() / s.norm()
    assert err.item() <= 1e-2


def test_overlap_and_baseline_bitwise_equal_full_size(comm):
    """P:L272 'C-Cube does not change the ordering of any computation'."""
    P, chunk = 8, 256 << 10
    comm(P, "single", chunk)
    _, _, a = _full_size(P, "single", "float32", "resnet50", chunk, overlap=True)
    _, _, b = _full_size(P, "single", "float32", "resnet50", chunk, overlap=False)
    for r in range(P):
        assert torch.equal(a[r], b[r])


@pytest.mark.parametrize("kind", ["single", "double"])
@pytest.mark.parametrize("gate", ["memop", "kernel"])
def test_gradient_queue_gates_each_layer(comm, monkeypatch, kind, gate):
    """a9: on a second stream, gradq_wait(l) then snapshot layer l's gradients; every
    snapshot must already hold the final reduced values.  Both gate
    mechanisms: the stream memory-op wait and the ld.acquire spin kernel
    (CCUBE_GATE_KERNEL=1, the one-process-per-GPU default without remote-write
    flush)."""
    if gate == "kernel":
        monkeypatch.setenv("CCUBE_GATE_KERNEL", "1")
    P, chunk = 8, 64 << 10
    comm(P, kind, chunk, channels=4)
    ends = workloads.layer_ends("resnet50")
    count = ends[-1]
    ts = device_inputs(P, count, "float32", layer_ends=ends)
    ccube.gradq_set_layers(ends)
    comm_stream = torch.cuda.Stream()
    comp = torch.cuda.Stream()
    comm_stream.wait_stream(torch.cuda.current_stream())
    comp.wait_stream(torch.cuda.current_stream())
    snaps = {}
    rank = 5
    with torch.cuda.stream(comm_stream):
        ccube.allreduce_tree_local(ts, stream=comm_stream)
    with torch.cuda.stream(comp):
        starts = [0] + ends[:-1]
        for l in range(len(ends)):
            ccube.gradq_wait_local(rank, l, stream=comp)
            snaps[l] = ts[rank][starts[l]:ends[l]].clone()
    torch.cuda.synchronize()
    final = ts[rank]
    for l in range(len(ends)):
        assert torch.equal(snaps[l], final[starts[l]:ends[l]]), f"layer {l} read before landing"


def test_landing_trace_in_order_and_c1_turnaround(comm):
    """Obs #3: chunks land in order per rank/tree/channel; C1 turns the first
    chunk around long before B (Fig 14(b))."""
    P, chunk, J = 8, 64 << 10, 4
    comm(P, "single", chunk, channels=J)
    count = 64 * chunk // 4
    K = 64
    trace = torch.zeros(P * 1 * K * J, dtype=torch.int64, device="cuda")
    ccube.set_trace(trace, K)
    ts = device_inputs(P, count, "float32")
    res = {}
    for overlap in (False, True):
        trace.zero_()
        ccube.set_overlap(overlap)
        ccube.allreduce_tree_local(ts)
        torch.cuda.synchronize()
        tr = trace.view(P, K, J).cpu().numpy().astype(np.int64)
        assert (tr > 0).all()
        for r in range(P):
            for j in range(J):
                assert np.all(np.diff(tr[r, :, j]) >= 0), (overlap, r, j)
        land = tr.max(axis=2)                    # a chunk has landed when all slices have
        t0 = tr.min()
        res[overlap] = (land[:, 0].max() - t0, land.max() - t0)
    ccube.set_trace(None, 0)
    turn_b, total_b = res[False]
    turn_c, total_c = res[True]
    assert turn_c * 4 < turn_b, res


# ---- rotated multi-tree set (reading R17) ---------------------------
@pytest.mark.parametrize("P", [2, 3, 4, 8])
@pytest.mark.parametrize("dtype", ["int32", "float32", "bfloat16"])
@pytest.mark.parametrize("overlap", [True, False])
@pytest.mark.parametrize("transport", ["pull", "push"])
def test_parity_rotated(comm, P, dtype, overlap, transport):
    """P trees, chunk c on tree c mod P: bit-exact vs the oracle definition, with
    several chunks per tree and a ragged tail."""
    chunk = 4096
    comm(P, "rotated", chunk, channels=2, overlap=overlap, transport=transport)
    E = chunk // arith.ELEM_SIZE[dtype]
    count = (2 * P + 3) * E + 13
    xs, outs = _run(P, "rotated", dtype, count, chunk)
    ref = oar.reference(xs, "rotated", chunk, dtype)[0]
    for r in range(P):
        assert np.array_equal(outs[r], ref), f"rank {r}"


def test_full_size_resnet50_rotated(comm):
    """ResNet-50 gradient set over the rotated set at P = 8 (auto channels): sampled
    chunks of every tree bit-exact vs the oracle, every rank identical."""
    P, chunk = 8, 256 << 10
    comm(P, "rotated", chunk)
    count, ends, ts = _full_size(P, "rotated", "float32", "resnet50", chunk)
    K = partition.num_chunks(count, chunk, 4)
    for c in sorted({0, 1, 2, 3, 4, 5, 6, 7, K - 2, K - 1, 200}):
        lo, hi, want = oracle_chunk(P, "rotated", chunk, "float32", count, c, layer_ends=ends)
        for r in (0, 5):
            assert np.array_equal(to_numpy(ts[r][lo:hi], "float32"), want), (c, r)
    for r in range(1, P):
        assert torch.equal(ts[r], ts[0])


def test_gradient_queue_gates_rotated(comm):
    """a9 with P trees: layer l needs #{c < LCT[l] : c mod P = t} chunks of tree t."""
    P, chunk = 8, 64 << 10
    comm(P, "rotated", chunk, channels=2)
    ends = workloads.layer_ends("resnet50")
    count = ends[-1]
    ts = device_inputs(P, count, "float32", layer_ends=ends)
    ccube.gradq_set_layers(ends)
    comm_stream, comp = torch.cuda.Stream(), torch.cuda.Stream()
    comm_stream.wait_stream(torch.cuda.current_stream())
    comp.wait_stream(torch.cuda.current_stream())
    snaps = {}
    rank = 3
    with torch.cuda.stream(comm_stream):
        ccube.allreduce_tree_local(ts, stream=comm_stream)
    with torch.cuda.stream(comp):
        starts = [0] + ends[:-1]
        for l in range(len(ends)):
            ccube.gradq_wait_local(rank, l, stream=comp)
            snaps[l] = ts[rank][starts[l]:ends[l]].clone()
    torch.cuda.synchronize()
    for l in range(len(ends)):
        assert torch.equal(snaps[l], ts[rank][starts[l]:ends[l]]), f"layer {l} read before landing"


# ---- fused SGD update at dequeue (reading R18) ----------------------
@pytest.mark.parametrize("P", [2, 4, 8])
@pytest.mark.parametrize("kind", ["single", "double", "rotated"])
@pytest.mark.parametrize("overlap", [True, False])
def test_fused_sgd_parity(comm, P, kind, overlap):
    """Every rank's weights become oracle.gradq.sgd_update(w, final, alpha) bit for
    bit (root: in its reduce; interior: in its broadcast; leaf: UPDATE task), and
    the gradients are still the oracle's fixed-order sum.  Ragged fp32 tail."""
    from oracle import gradq as ogq
    chunk = 4096
    comm(P, kind, chunk, channels=2, overlap=overlap)
    E = chunk // 4
    count = 7 * E + 13
    ws0 = [inputs.gradients(r + 100, count, "float32") for r in range(P)]
    ws = [to_torch(w, "float32").cuda() for w in ws0]
    alpha = 0.013
    ccube.gradq_set_sgd(ws, alpha)
    xs, outs = _run(P, kind, "float32", count, chunk)
    ref = oar.reference(xs, kind, chunk, "float32")[0]
    for r in range(P):
        assert np.array_equal(outs[r], ref), f"grads rank {r}"
        want = ogq.sgd_update(ws0[r], ref, alpha)
        assert np.array_equal(to_numpy(ws[r], "float32"), want), f"weights rank {r}"
    ccube.gradq_set_sgd(None)


def test_fused_sgd_gate_waits_for_weights(comm):
    """With the fused update the gate opens once the layer's weights are updated."""
    P, chunk, rank = 8, 64 << 10, 5
    comm(P, "double", chunk, channels=2)
    ends = workloads.layer_ends("resnet50")
    count = ends[-1]
    ts = device_inputs(P, count, "float32", layer_ends=ends)
    ws = device_inputs(P, count, "float32", seed=99)
    ccube.gradq_set_layers(ends)
    ccube.gradq_set_sgd(ws, 0.01)
    comm_stream, comp = torch.cuda.Stream(), torch.cuda.Stream()
    comm_stream.wait_stream(torch.cuda.current_stream())
    comp.wait_stream(torch.cuda.current_stream())
    snaps = {}
    with torch.cuda.stream(comm_stream):
        ccube.allreduce_tree_local(ts, stream=comm_stream)
    with torch.cuda.stream(comp):
        starts = [0] + ends[:-1]
        for l in range(len(ends)):
            ccube.gradq_wait_local(rank, l, stream=comp)
            snaps[l] = ws[rank][starts[l]:ends[l]].clone()
    torch.cuda.synchronize()
    for l in range(len(ends)):
        assert torch.equal(snaps[l], ws[rank][starts[l]:ends[l]]), f"layer {l} weights early"
    ccube.gradq_set_sgd(None)


def test_fused_sgd_rejects_non_fp32(comm):
    comm(4, "single", 4096)
    ws = [torch.zeros(4096, device="cuda") for _ in range(4)]
    ccube.gradq_set_sgd(ws, 0.1)
    ts = [torch.zeros(2048, dtype=torch.bfloat16, device="cuda") for _ in range(4)]
    with pytest.raises(ccube.CCubeError) as e:
        ccube.allreduce_tree_local(ts)
    assert e.value.code == ccube.ERR_INVALID_ARG
    ccube.gradq_set_sgd(None)


@pytest.mark.parametrize("P", [2, 3, 5, 8])
@pytest.mark.parametrize("kind", ["single", "double", "rotated"])
@pytest.mark.parametrize("dtype", ["int32", "float32", "bfloat16"])
@pytest.mark.parametrize("transport", ["pull", "push"])
def test_parity_tma_datapath(comm, P, kind, dtype, transport):
    """The TMA datapath (cp.async.bulk shared-memory ring, consumer warps combine from
    shared memory) is bit-exact to the oracle: several chunks, ragged tail (< 16 B)
    and slices longer than one ring stage (8 KB) at 2 channels."""
    chunk = 48 * 1024
    comm(P, kind, chunk, channels=2, transport=transport)
    ccube.set_datapath("tma")
    assert ccube.get_info()["datapath"] == 1
    E = chunk // arith.ELEM_SIZE[dtype]
    count = 5 * E + 7 if dtype == "bfloat16" else 5 * E + 3
    xs, outs = _run(P, kind, dtype, count, chunk)
    assert ccube.get_info()["last_tma"] == 1
    ref = oar.reference(xs, kind, chunk, dtype)[0]
    for r in range(P):
        assert np.array_equal(outs[r], ref), f"rank {r}"


def test_parity_full_size_tma(comm):
    """configs[1] in the bench's launch configuration (P = 8, single tree, C1, auto
    channels) on the TMA datapath: sampled chunks bit-exact vs the oracle, every rank
    identical."""
    P, chunk = 8, 256 << 10
    comm(P, "single", chunk)
    ccube.set_datapath("tma")
    count, ends, ts = _full_size(P, "single", "float32", "resnet50", chunk)
    K = partition.num_chunks(count, chunk, 4)
    for c in (0, 1, 200, K - 2, K - 1):
        lo, hi, want = oracle_chunk(P, "single", chunk, "float32", count, c, layer_ends=ends)
        for r in (0, 2, 7):
            assert np.array_equal(to_numpy(ts[r][lo:hi], "float32"), want), (c, r)
    for r in range(1, P):
        assert torch.equal(ts[r], ts[0])


@pytest.mark.parametrize("order", [1, 2])
@pytest.mark.parametrize("kind", ["single", "double", "rotated"])
@pytest.mark.parametrize("sgd", [False, True])
def test_parity_task_order(comm, monkeypatch, order, kind, sgd):
    """CCUBE_TASK_ORDER only moves tasks between blocks (which tasks share an SM);
    the results stay bit-exact, with and without the fused update's UPDATE tasks."""
    monkeypatch.setenv("CCUBE_TASK_ORDER", str(order))
    P, chunk, count = 8, 4096, 20_011
    comm(P, kind, chunk, channels=3)
    xs = [inputs.gradients(r, count, "float32", seed=11) for r in range(P)]
    ts = [to_torch(x, "float32").cuda() for x in xs]
    if sgd:
        from oracle import gradq as ogq
        ws = [torch.ones(count, device="cuda") for _ in range(P)]
        ccube.gradq_set_sgd(ws, 0.5)
    ccube.allreduce_tree_local(ts)
    torch.cuda.synchronize()
    ref = oar.reference(xs, kind, chunk, "float32")[0]
    for t in ts:
        np.testing.assert_array_equal(to_numpy(t, "float32"), ref)
    if sgd:
        want = ogq.sgd_update(np.ones(count, np.float32), ref, 0.5)
        for w in ws:
            np.testing.assert_array_equal(to_numpy(w, "float32"), want)
        ccube.gradq_set_sgd(None)


# ---- placement (reading R19) ---------------------------------------------------------
def _placed_run(P, kind, dtype, perm, count, chunk, channels=3, overlap=True, seed=21, xs=None):
    ccube.set_placement(perm)
    try:
        ccube.init_loopback(P, kind, chunk)
        try:
            ccube.set_channels(channels)
            ccube.set_overlap(overlap)
            if xs is None:
                xs = [inputs.gradients(r, count, dtype, seed=seed) for r in range(P)]
            ts = [to_torch(x, dtype).cuda() for x in xs]
            ccube.allreduce_tree_local(ts)
            torch.cuda.synchronize()
            return xs, [to_numpy(t, dtype) for t in ts]
        finally:
            ccube.finalize()
    finally:
        ccube.set_placement(None)


@pytest.mark.parametrize("P", [3, 4, 8])
@pytest.mark.parametrize("kind", ["single", "double", "rotated"])
@pytest.mark.parametrize("dtype", ["int32", "float32", "bfloat16"])
@pytest.mark.parametrize("overlap", [True, False])
def test_parity_placement(P, kind, dtype, overlap):
    """A placed tree set (position v on rank perm[v]) is bit-exact to the oracle
    with the same permutation; ragged tail, several chunks per tree."""
    perm = [int(v) for v in np.random.default_rng(P + 7).permutation(P)]
    chunk = 4096
    count = 9 * (chunk // 4) + 5
    xs, outs = _placed_run(P, kind, dtype, perm, count, chunk, overlap=overlap)
    ref = oar.reference(xs, kind, chunk, dtype, perm=perm)[0]
    for r in range(P):
        assert np.array_equal(outs[r].view(np.uint8), ref.view(np.uint8)), f"rank {r}"


def test_placement_order_pin_gpu():
    """The hand-derived pin of tests/test_placement.py on the GPU: identity 1.0,
    reversal 0.0 for x = (1, 2^24, 1, -2^24)."""
    xs = [np.array([v] * 4, np.float32) for v in (1.0, 2.0 ** 24, 1.0, -2.0 ** 24)]
    _, outs = _placed_run(4, "single", "float32", [0, 1, 2, 3], 4, 16, channels=1, xs=xs)
    assert all(o[0] == 1.0 for o in outs)
    _, outs = _placed_run(4, "single", "float32", [3, 2, 1, 0], 4, 16, channels=1, xs=xs)
    assert all(o[0] == 0.0 for o in outs)


def test_parity_placement_full_size_resnet50():
    """ResNet-50 gradient set, P = 8, double tree, a planned placement for a matrix
    with two slow pairs, bench launch configuration (auto channels)."""
    from oracle import placement as opl
    P = 8
    bw = np.full((P, P), 100.0)
    bw[0, 4] = bw[4, 0] = bw[3, 7] = bw[7, 3] = 10.0
    perm = ccube.plan_placement(bw, "double")
    assert perm == opl.plan(P, "double", bw) and perm != list(range(P))
    ends = workloads.layer_ends("resnet50")
    count = ends[-1]
    xs = [inputs.gradients(r, count, "float32", layer_ends=ends) for r in range(P)]
    _, outs = _placed_run(P, "double", "float32", perm, count, 256 << 10, channels=0, xs=xs)
    ref = oar.reference(xs, "double", 256 << 10, "float32", perm=perm)[0]
    for r in range(P):
        assert np.array_equal(outs[r], ref), f"rank {r}"


@pytest.mark.parametrize("kind", ["single", "double"])
def test_max_size_1gib_ragged(comm, kind):
    """configs[4]'s largest message (1 GiB per rank, fp32) minus a ragged tail of 37
    elements, P = 8, 256 KiB chunks (K = 4096). Each rank's buffer is its seeded
    generator block of B = 2^20 + 7 elements repeated (B is not a multiple of the chunk,
    so no two chunks see the same data); sampled chunks bit-exact vs the oracle's fold
    on the same values (first, the ragged last, random), every rank identical."""
    from oracle import trees as otrees

    P, chunk, B = 8, 256 << 10, (1 << 20) + 7
    count = (1 << 28) - 37
    comm(P, kind, chunk)
    base = [inputs.gradients(r, B, "float32", seed=11) for r in range(P)]
    ts = []
    for r in range(P):
        b = torch.from_numpy(base[r]).cuda()
        ts.append(b.repeat((count + B - 1) // B)[:count].contiguous())
    ccube.allreduce_tree_local(ts)
    torch.cuda.synchronize()
    K = partition.num_chunks(count, chunk, 4)
    assert K == 4096
    trees = otrees.trees(P, kind)
    rng = np.random.default_rng(1)
    for c in sorted({0, 1, K - 2, K - 1, *rng.integers(0, K, 6).tolist()}):
        lo, hi = partition.chunk_range(c, count, chunk, 4)
        idx = np.arange(lo, hi) % B
        tree = trees[partition.tree_of_chunk(c, len(trees))]
        want = oar.fold([x[idx] for x in base], tree, tree.root, "float32")
        for r in (0, 7):
            assert np.array_equal(to_numpy(ts[r][lo:hi], "float32"), want), (c, r)
    for r in range(1, P):
        assert torch.equal(ts[r], ts[0])


# ---- IEEE corner cases: inputs.special ---------------------------------
def _run_special(P, kind, dtype, count, chunk):
    xs = [inputs.special(r, count, dtype) for r in range(P)]
    ts = [to_torch(x, dtype).cuda() for x in xs]
    ccube.allreduce_tree_local(ts)
    torch.cuda.synchronize()
    return xs, [to_numpy(t, dtype) for t in ts]


@pytest.mark.parametrize("P", [4, 8])
@pytest.mark.parametrize("kind", ["single", "double", "rotated"])
@pytest.mark.parametrize("dtype", ["int32", "float32", "bfloat16"])
@pytest.mark.parametrize("overlap", [True, False])
@pytest.mark.parametrize("transport", ["pull", "push"])
@pytest.mark.parametrize("datapath", ["lsu", "tma"])
def test_parity_special_values(comm, P, kind, dtype, overlap, transport, datapath):
    """Subnormals, +-0, near-max values, the normal/subnormal boundary, exact
    cancellation and int32 extremes (inputs.special): bit-exact vs the oracle on
    every tree, B and C1, both edge transports and both datapaths, ragged tail.  A
    build with -ftz=true, a contracted FMA or a wrong signed-zero rule fails here."""
    chunk = 4096
    comm(P, kind, chunk, channels=3, overlap=overlap, transport=transport)
    ccube.set_datapath(datapath)
    E = chunk // arith.ELEM_SIZE[dtype]
    count = 7 * E + 13
    xs, outs = _run_special(P, kind, dtype, count, chunk)
    ref = oar.reference(xs, kind, chunk, dtype)[0]
    for r in range(P):
        assert np.array_equal(outs[r], ref), f"rank {r}"


@pytest.mark.parametrize("dtype", ["float32", "bfloat16"])
def test_device_keeps_subnormals_and_signed_zeros(comm, dtype):
    """Reading R3 observed on the device: where every rank holds a subnormal the
    result is a nonzero subnormal (no FTZ/DAZ), where every rank holds -0 it is -0,
    where the signs mix it is +0."""
    P, chunk = 8, 1 << 16
    comm(P, "double", chunk)
    count = 200_003
    xs, outs = _run_special(P, "double", dtype, count, chunk)
    f = arith.to_float64(outs[3], dtype)
    cls = inputs.special_class(0, count)
    sub = cls == 2
    assert (f[sub] != 0).mean() > 0.9
    assert (np.abs(f[sub]) < 2.0 ** -126).all()
    z = cls == 3
    vals = np.stack([arith.to_float64(x, dtype)[z] for x in xs])
    all_neg = np.signbit(vals).all(axis=0)
    assert (f[z] == 0).all()
    assert np.array_equal(np.signbit(f[z]), all_neg) and all_neg.any() and (~all_neg).any()


_R50 = {}


def _resnet50_reference(P, kind, chunk):
    """The oracle's whole-buffer result for the ResNet-50 set (cached per tree kind:
    B and C1 share it)."""
    if "xs" not in _R50:
        ends = workloads.layer_ends("resnet50")
        _R50["xs"] = [inputs.gradients(r, ends[-1], "float32", layer_ends=ends)
                      for r in range(P)]
    if kind not in _R50:
        _R50[kind] = oar.reference(_R50["xs"], kind, chunk, "float32")[0]
    return _R50[kind]


@pytest.mark.parametrize("kind", ["single", "double", "rotated"])
@pytest.mark.parametrize("overlap", [True, False])
def test_full_size_resnet50_fp32_whole_buffer(comm, kind, overlap):
    """configs[1] at full size in the bench's launch configuration (P = 8, 256 KiB
    chunks, auto channels): EVERY element of every rank's buffer bit-exact vs the
    oracle's definition (the whole 25.6M-element fold)."""
    P, chunk = 8, 256 << 10
    comm(P, kind, chunk)
    ends = workloads.layer_ends("resnet50")
    count = ends[-1]
    ts = device_inputs(P, count, "float32", layer_ends=ends)
    ccube.set_overlap(overlap)
    ccube.allreduce_tree_local(ts)
    torch.cuda.synchronize()
    ref = _resnet50_reference(P, kind, chunk)
    for r in range(P):
        got = to_numpy(ts[r], "float32")
        assert np.array_equal(got.view(np.uint32), ref.view(np.uint32)), \
            f"rank {r}: {int((got.view(np.uint32) != ref.view(np.uint32)).sum())} elements differ"


# ---- LL protocol (one-chunk calls: flag-in-data) -------------------------
@pytest.mark.parametrize("P", [2, 3, 4, 5, 8])
@pytest.mark.parametrize("kind", ["single", "double", "rotated"])
@pytest.mark.parametrize("dtype", ["int32", "float32", "bfloat16"])
@pytest.mark.parametrize("count", [1, 3, 1023, 20_001])
def test_parity_ll(comm, P, kind, dtype, count):
    """A one-chunk message runs the LL kernel: bit-exact vs the oracle (tree 0's fold)
    for every tree kind, odd bf16 counts included."""
    chunk = 256 << 10
    comm(P, kind, chunk)
    xs, outs = _run(P, kind, dtype, count, chunk)
    assert ccube.get_info()["last_ll"] == 1
    ref = oar.reference(xs, kind, chunk, dtype)[0]
    for r in range(P):
        assert np.array_equal(outs[r], ref), f"rank {r}"


@pytest.mark.parametrize("dtype", ["float32", "bfloat16"])
def test_ll_special_values_and_max_size(comm, dtype):
    """IEEE corner cases through the LL kernel, at its largest message (256 KiB)."""
    P, chunk = 8, 256 << 10
    comm(P, "double", chunk)
    count = (256 << 10) // arith.ELEM_SIZE[dtype]
    xs, outs = _run_special(P, "double", dtype, count, chunk)
    assert ccube.get_info()["last_ll"] == 1
    ref = oar.reference(xs, "double", chunk, dtype)[0]
    for r in range(P):
        assert np.array_equal(outs[r], ref), f"rank {r}"


def test_ll_equals_chunked_and_interleaves(comm):
    """LL and chunked calls alternate on one communicator (epochs and counters stay
    consistent); both give the same bits as the oracle; LL off runs the chunked
    kernel for the same one-chunk size."""
    P, chunk = 8, 64 << 10
    comm(P, "double", chunk)
    for it, count in enumerate([100, 50_000, 7, 16_384, 70_001, 1]):
        ccube.set_protocol(it % 3 != 2)
        xs, outs = _run(P, "double", "float32", count, chunk, seed=300 + it)
        ll = count * 4 <= chunk and it % 3 != 2
        assert ccube.get_info()["last_ll"] == int(ll), (it, count)
        ref = oar.reference(xs, "double", chunk, "float32")[0]
        for r in range(P):
            assert np.array_equal(outs[r], ref), (it, r)


def test_ll_gate_opens_after_landing(comm):
    """ccube_gradq_wait after an LL call: every layer's snapshot holds final values."""
    P, chunk = 8, 256 << 10
    comm(P, "single", chunk)
    count = 60_000
    ends = [1000, 30_000, count]
    ts = device_inputs(P, count, "float32")
    ccube.gradq_set_layers(ends)
    cs, comp = torch.cuda.Stream(), torch.cuda.Stream()
    cs.wait_stream(torch.cuda.current_stream())
    comp.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(cs):
        ccube.allreduce_tree_local(ts, stream=cs)
    snaps = []
    with torch.cuda.stream(comp):
        lo = 0
        for l, hi in enumerate(ends):
            ccube.gradq_wait_local(7, l, stream=comp)
            snaps.append(ts[7][lo:hi].clone())
            lo = hi
    torch.cuda.synchronize()
    assert ccube.get_info()["last_ll"] == 1
    lo = 0
    for s, hi in zip(snaps, ends):
        assert torch.equal(s, ts[7][lo:hi])
        lo = hi


@pytest.mark.parametrize("P,kind", [(8, "single"), (8, "double"), (4, "single"), (2, "single")])
@pytest.mark.parametrize("overlap", [True, False])
def test_parity_split_heads(comm, monkeypatch, P, kind, overlap):
    """CCUBE_SPLIT_HEADS=1: the pipeline's head tasks on two CTAs per channel, the
    halves publishing a monotone max of their joint progress — bit-exact vs the
    oracle, several chunks, ragged tail, auto channels."""
    monkeypatch.setenv("CCUBE_SPLIT_HEADS", "1")
    chunk = 64 << 10
    comm(P, kind, chunk, overlap=overlap)
    count = 9 * chunk // 4 + 77
    xs, outs = _run(P, kind, "float32", count, chunk)
    ref = oar.reference(xs, kind, chunk, "float32")[0]
    for r in range(P):
        assert np.array_equal(outs[r], ref), f"rank {r}"

"""Host-side checks of the C ABI that need no GPU: exports, trees, validation,
and the multi-process bootstrap (config agreement over a gloo allgather)."""

import os
import re
import socket

import pytest

from oracle import trees as otrees
from paper_conf_hpca_sanghoonsk23_b200 import ccube

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _header_functions():
    src = open(os.path.join(ROOT, "include", "ccube.h")).read()
    return sorted(set(re.findall(r"CCUBE_API\s+[\w\s\*]+?\b(ccube_\w+)\s*\(", src)))


def test_library_exports_every_header_symbol():
    L = ccube.lib()
    names = _header_functions()
    assert len(names) >= 15
    for n in names:
        assert hasattr(L, n), n
    assert sorted(ccube.EXPORTS) == names


@pytest.mark.parametrize("P", range(1, 17))
@pytest.mark.parametrize("kind,tree", [("single", 0), ("double", 0), ("double", 1)])
def test_library_trees_match_oracle(P, kind, tree):
    """The library builds tree 0 top-down (children rule) and tree 1 by renaming;
    the oracle builds them bottom-up (parent rule): both must agree (R1)."""
    want = otrees.trees(P, kind)[tree].parent
    assert ccube.tree_parents(P, kind, tree) == list(want)


def test_tree_parents_rejects_bad_args():
    with pytest.raises(ccube.CCubeError) as e:
        ccube.tree_parents(4, "single", 1)
    assert e.value.code == ccube.ERR_INVALID_ARG


def test_calls_before_init_fail_cleanly():
    for fn, args in [(ccube.set_overlap, (1,)), (ccube.set_channels, (4,)),
                     (ccube.set_datapath, ("tma",)), (ccube.set_datapath, ("auto",)),
                     (ccube.gradq_set_layers, ([1, 2],)), (ccube.finalize, ())]:
        with pytest.raises(ccube.CCubeError) as e:
            fn(*args)
        assert e.value.code == ccube.ERR_NOT_INITIALIZED
    assert "ccube_init" in ccube.last_error()
    assert ccube.get_info()["initialized"] == 0


@pytest.mark.parametrize("kwargs,code", [
    (dict(world_size=9), ccube.ERR_UNSUPPORTED),
    (dict(world_size=0), ccube.ERR_INVALID_ARG),
    (dict(world_size=4, nlocal=3), ccube.ERR_INVALID_ARG),
    (dict(world_size=4, chunk_bytes=1000), ccube.ERR_INVALID_ARG),
    (dict(world_size=4, chunk_bytes=16 * 7 + 8), ccube.ERR_INVALID_ARG),   # not a multiple of 16
    (dict(world_size=4, rank=1), ccube.ERR_INVALID_ARG),
])
def test_init_validation(kwargs, code):
    with pytest.raises(ccube.CCubeError) as e:
        ccube.init(**kwargs)
    assert e.value.code == code
    assert ccube.get_info()["initialized"] == 0


def test_init_without_gpu_reports_cuda_error():
    import torch
    if torch.cuda.is_available():
        pytest.skip("this check is for GPU-less hosts")
    for _ in range(2):  # state is reset after a failed init
        with pytest.raises(ccube.CCubeError) as e:
            ccube.init_loopback(4)
        assert e.value.code == ccube.ERR_CUDA
    assert ccube.get_info()["initialized"] == 0


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _bootstrap_worker(rank, world, port, chunk_for_rank, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_hpca_sanghoonsk23_b200 import ccube as cc
    try:
        cc.init(world, rank=rank, nlocal=1, device=0, tree="double",
                chunk_bytes=chunk_for_rank[rank], pg=dist.group.WORLD)
        q.put((rank, 0, ""))
        cc.finalize()
    except cc.CCubeError as e:
        q.put((rank, e.code, str(e)))
    dist.destroy_process_group()


def _run_bootstrap(chunks):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_bootstrap_worker, args=(r, 2, port, chunks, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = sorted(q.get(timeout=120) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    return out


def test_gloo_bootstrap_agreement_ws2():
    """world_size 2 over gloo: the config-agreement allgather succeeds on both ranks;
    then CUDA setup fails on a GPU-less host (or refuses two processes on one GPU)."""
    out = _run_bootstrap([256 << 10, 256 << 10])
    for rank, code, msg in out:
        assert code in (ccube.SUCCESS, ccube.ERR_CUDA, ccube.ERR_UNSUPPORTED), msg
        assert "disagree" not in msg


def test_gloo_bootstrap_detects_mismatch_ws2():
    out = _run_bootstrap([256 << 10, 128 << 10])
    for rank, code, msg in out:
        assert code == ccube.ERR_INVALID_ARG, msg
        assert "disagree" in msg

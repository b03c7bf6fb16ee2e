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


# ---- launch geometry is a collective decision -----------------------

def _py_tasks(P, kind, nlocal, proc, J, overlap):
    """Independent restatement of the task table: per rank and tree, UP on J channels,
    DOWN on J channels at interior nodes (and at the root in B); a rank that is a
    pulled leaf (same process as its parent) in any tree adds one leaf-group CTA."""
    T = {"single": 1, "double": 2, "rotated": P}[kind]
    n = 0
    for r in range(proc * nlocal, (proc + 1) * nlocal):
        pulled = False
        for t in range(T):
            par = ccube.tree_parents(P, kind, t)
            nch = sum(1 for u in range(P) if par[u] == r)
            root = par[r] < 0
            if not root and nch == 0 and par[r] // nlocal == r // nlocal:
                pulled = True
                continue
            n += J
            if nch > 0 and (not root or not overlap):
                n += J
        n += 1 if pulled else 0
    return n


def _py_jmax(nbytes, chunk):
    first = min(nbytes, chunk)
    units = -(-first // 2048)
    per = 1 if nbytes >= 16 * chunk else 2
    return max(units // per, 1)


SIZES = [1 << 10, 1 << 20, 4 << 20, 102_228_128, 1 << 30]


@pytest.mark.parametrize("P", range(2, 9))
@pytest.mark.parametrize("kind", ["single", "double", "rotated"])
@pytest.mark.parametrize("overlap", [0, 1])
def test_plan_launch_every_rank_agrees(P, kind, overlap):
    """One process per GPU: every rank gets the same J for every size (so both ends of
    an edge slice chunks alike), J is the largest whose busiest process fits the cap,
    and no process exceeds the cap."""
    cap = 296   # 2 CTAs x 148 SMs (B200, 320-thread CTAs)
    for nbytes in SIZES:
        got = [ccube.plan_launch(P, kind, 1, r, nbytes, 256 << 10, overlap, 0, cap)
               for r in range(P)]
        Js = {j for j, _, _ in got}
        assert len(Js) == 1, (nbytes, got)
        J = Js.pop()
        tasks = [_py_tasks(P, kind, 1, r, J, overlap) for r in range(P)]
        assert [n for _, n, _ in got] == tasks
        assert all(m == max(tasks) for _, _, m in got)
        assert max(tasks) <= cap
        # J is maximal: one more channel would overflow the busiest process, or the
        # per-chunk unit cap binds
        jmax = min(_py_jmax(nbytes, 256 << 10), 128)
        assert J == jmax or max(_py_tasks(P, kind, 1, r, J + 1, overlap)
                                for r in range(P)) > cap


def test_per_rank_rule_would_disagree():
    """The round-1 rule (J from this process's own tasks) gives the roots of the
    double tree at P=8, C1, >= 16 chunks a different J than the other ranks — the
    hang the collective rule removes."""
    P, cap, nbytes = 8, 296, 102_228_128
    own = []
    for r in range(P):
        J = 1
        while J < 128 and _py_tasks(P, "double", 1, r, J + 1, 1) <= cap:
            J += 1
        own.append(min(J, _py_jmax(nbytes, 256 << 10)))
    assert len(set(own)) > 1, own
    lib = {ccube.plan_launch(P, "double", 1, r, nbytes, 256 << 10, 1, 0, cap)[0]
           for r in range(P)}
    assert lib == {min(own)}


def test_plan_launch_loopback_and_explicit():
    # loopback: one process hosts every rank
    j, n, m = ccube.plan_launch(8, "single", 8, 0, 102_228_128, 256 << 10, 1, 0, 296)
    assert n == m == _py_tasks(8, "single", 8, 0, j, 1) <= 296
    assert j == 41   # 7 J + 4 leaf-group CTAs (one per leaf rank) <= 296
    # the double tree: 14 J + 8 <= 296 -> 20; the rotated set at P = 8: 56 J + 8 -> 5
    # (round 1 spent one CTA per pulled leaf and tree: 56 J + 32 -> 4)
    assert ccube.plan_launch(8, "double", 8, 0, 102_228_128, 256 << 10, 1, 0, 296)[0] == 20
    assert ccube.plan_launch(8, "rotated", 8, 0, 102_228_128, 256 << 10, 1, 0, 296)[0] == 5
    # explicit channels are returned as given
    assert ccube.plan_launch(4, "double", 1, 2, 1 << 20, 0, 1, 7, 296)[0] == 7
    with pytest.raises(ccube.CCubeError) as e:
        ccube.plan_launch(4, "double", 3, 0, 1 << 20, 0, 1, 0, 296)
    assert e.value.code == ccube.ERR_INVALID_ARG


def _env_worker(rank, world, port, env, q):
    os.environ.update(env[rank])
    _bootstrap_worker(rank, world, port, [256 << 10] * world, q)


def test_gloo_bootstrap_detects_launch_setting_mismatch_ws2():
    """CCUBE_CHANNELS differs between the two processes: both refuse at init."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    env = [{"CCUBE_CHANNELS": "8"}, {"CCUBE_CHANNELS": "16"}]
    procs = [ctx.Process(target=_env_worker, args=(r, 2, port, env, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = sorted(q.get(timeout=120) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    for rank, code, msg in out:
        assert code == ccube.ERR_INVALID_ARG, msg
        assert "launch settings" in msg

"""Host-side checks of the measurement tools (no GPU): the alpha-beta fit recovers
known constants, the all-cores oracle pool gives the single-core replay's bits, and
the NVLink counter summary parses ncu's CSV layout."""

import json
import math
import os
import subprocess
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))


def test_model_fit_recovers_known_constants(tmp_path):
    """Synthetic sweep from T = t0 + 2D alpha + steps * beta * C (plus LL rows):
    the anchored non-negative fit returns t0, alpha and beta."""
    import model_fit
    t0, alpha, beta = 4.0, 2.5, 1 / 700e3      # us, us/hop, us/byte
    rows = []
    for P in (2, 4, 8):
        D = model_fit.DEPTH[P]
        for nbytes in [1 << k for k in range(10, 31, 2)]:
            for mode in ("C1", "B"):
                r = {"P": P, "tree": "single", "mode": mode, "bytes": nbytes,
                     "chunk_bytes": 256 << 10, "protocol": "chunked"}
                n, nC = model_fit.design(r, 1, D)
                r["us"] = t0 + 2 * D * alpha + beta * nC
                rows.append(r)
            rows.append({"P": P, "tree": "single", "mode": "C1", "bytes": nbytes,
                         "chunk_bytes": 256 << 10, "protocol": "ll",
                         "us": 3.0 + 2 * D * 0.5})
    path = tmp_path / "sizes.jsonl"
    path.write_text("\n".join(json.dumps(r) for r in rows))
    out = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "model_fit.py"), str(path)],
                         capture_output=True, text=True, check=True).stdout
    d = json.loads(out)
    assert math.isclose(d["t0_us"], t0, rel_tol=1e-3, abs_tol=0.05)
    assert math.isclose(d["alpha_us_per_hop"], alpha, rel_tol=1e-2)
    assert math.isclose(d["ll"]["alpha_us_per_hop"], 0.5, rel_tol=1e-2)
    for f in d["fits"]:
        assert math.isclose(f["beta_us_per_byte"], beta, rel_tol=1e-3)
        for s in f["sizes"]:
            assert math.isclose(s["model_B_us"], s["measured_B_us"], rel_tol=1e-3)


def test_oracle_pool_matches_single_core_replay():
    """bench.OraclePool splits the chunks over processes; timing aside, the split must
    not change the work: every range replays exactly like the whole sample."""
    import bench
    from oracle import allreduce as oar
    from oracle import arith
    P, tree, chunk = 4, "double", 16 << 10
    xs, nbytes = bench.oracle_inputs(P, "float32", "resnet50", chunk, 12)
    whole, _ = oar.replay(xs, tree, chunk, "float32")
    E = chunk // arith.ELEM_SIZE["float32"]
    parts = []
    for c0, c1 in [(0, 4), (4, 8), (8, 12)]:       # ranges start at multiples of T = 2
        sub = [x[c0 * E:c1 * E] for x in xs]
        parts.append(oar.replay(sub, tree, chunk, "float32")[0][0])
    assert np.array_equal(np.concatenate(parts), whole[0])
    pool = bench.OraclePool(P, tree, "float32", "resnet50", chunk, 3, True, cores=2)
    try:
        assert pool.cores == 2 and pool.nch == 6
        assert pool.run() > 0
    finally:
        pool.close()


def test_nvlink_summary_parses_ncu_csv(tmp_path):
    import nvlink_summary
    csv_text = "\n".join([
        '"==PROF== log"',
        '"ID","Process ID","Process Name","Host Name","Kernel Name","Context","Stream",'
        '"Block Size","Grid Size","Device","CC","Section Name","Metric Name","Metric Unit",'
        '"Metric Value"',
        '"0","1","python","h","tree_allreduce_kernel","1","7","(256,1,1)","(291,1,1)","0","10.0",'
        '"Command line profiler metrics","gpu__time_duration.sum","usecond","200"',
        '"0","1","python","h","tree_allreduce_kernel","1","7","(256,1,1)","(291,1,1)","0","10.0",'
        '"Command line profiler metrics","nvltx__bytes.sum","Mbyte","100"',
        '"0","1","python","h","tree_allreduce_kernel","1","7","(256,1,1)","(291,1,1)","0","10.0",'
        '"Command line profiler metrics","nvlrx__bytes.sum","Mbyte","50"',
    ])
    p = tmp_path / "nv.csv"
    p.write_text(csv_text)
    (row,) = nvlink_summary.parse(str(p))
    assert math.isclose(row["us"], 200.0)
    assert math.isclose(row["nvltx__bytes_gbs"], 100e6 / 200e-6 / 1e9)
    assert math.isclose(row["nvlrx__bytes_gbs"], 50e6 / 200e-6 / 1e9)

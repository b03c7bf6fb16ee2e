"""A small loopback workload for compute-sanitizer (SURVEY §4 layer 2, §5): P = 4
ranks, every dtype, single / double / rotated tree, B and C1, the chunked kernel
(several chunks, ragged tail, both datapaths), the LL kernel (one chunk) and the
gradient-queue gate kernel; every result checked against a plain fp64/int64 sum
bound so a corrupting access also fails here.

    compute-sanitizer --tool memcheck  python tools/sanitize_case.py
    compute-sanitizer --tool racecheck python tools/sanitize_case.py
    compute-sanitizer --tool synccheck python tools/sanitize_case.py
"""
import os
import sys

os.environ.setdefault("CCUBE_GATE_KERNEL", "1")   # exercise the spin-gate kernel too

import torch  # noqa: E402

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_sanghoonsk23_b200 import ccube  # noqa: E402


def main():
    torch.cuda.set_device(0)
    P, chunk = 4, 8192
    checks = 0
    for kind in ("single", "double", "rotated"):
        ccube.init_loopback(P, kind, chunk)
        try:
            ccube.set_channels(3)
            for dt in (torch.float32, torch.bfloat16, torch.int32):
                for count, datapath, overlap in ((7 * chunk // 4 + 5, "lsu", True),
                                                 (7 * chunk // 4 + 5, "tma", False),
                                                 (1001, "lsu", True)):      # one chunk: LL
                    ccube.set_datapath(datapath)
                    ccube.set_overlap(overlap)
                    g = torch.Generator(device="cuda").manual_seed(count)
                    if dt == torch.int32:
                        xs = [torch.randint(-1000, 1000, (count,), device="cuda", generator=g,
                                            dtype=torch.int32) for _ in range(P)]
                    else:
                        xs = [torch.randn(count, device="cuda", generator=g).to(dt)
                              for _ in range(P)]
                    want = sum(x.double() for x in xs)
                    ccube.gradq_set_layers([count // 2, count])
                    ccube.allreduce_tree_local(xs)
                    s = torch.cuda.Stream()
                    ccube.gradq_wait_local(1, 1, stream=s)
                    torch.cuda.synchronize()
                    tol = 0 if dt == torch.int32 else (1e-5 if dt == torch.float32 else 5e-2)
                    for x in xs:
                        err = (x.double() - want).abs().max().item()
                        assert err <= tol * (1 + want.abs().max().item()), (kind, dt, count, err)
                    checks += 1
        finally:
            ccube.finalize()
    print(f"sanitize_case: {checks} AllReduce checks passed")


if __name__ == "__main__":
    main()

"""Summarise tools/nvlink_counters.sh's per-process ncu CSVs: per rank (process) and
launch, NVLink tx/rx and HBM read/write bytes and GB/s over the kernel's duration."""
import csv
import json
import sys
from collections import defaultdict


def parse(path):
    rows = list(csv.reader(open(path)))
    start = next((i for i, r in enumerate(rows) if "Metric Name" in r), None)
    if start is None:
        return []
    h = rows[start]
    ki, idi = h.index("Kernel Name"), h.index("ID")
    mi, vi, ui = h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit")
    launches = defaultdict(dict)
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1, "us": 1e3,
             "usecond": 1e3, "msecond": 1e6, "nsecond": 1}
    for r in rows[start + 1:]:
        if len(r) <= vi:
            continue
        v = float(r[vi].replace(",", "")) * scale.get(r[ui], 1)
        launches[r[idi]][r[mi]] = v
        launches[r[idi]]["kernel"] = r[ki][:60]
    out = []
    for lid, m in launches.items():
        t = m.get("gpu__time_duration.sum", 0) / 1e9
        d = {"id": lid, "kernel": m["kernel"], "us": t * 1e6}
        for k in ("nvltx__bytes.sum", "nvlrx__bytes.sum", "dram__bytes_read.sum",
                  "dram__bytes_write.sum"):
            d[k] = m.get(k)
            d[k.replace(".sum", "_gbs")] = (m[k] / t / 1e9) if t and m.get(k) is not None else None
        out.append(d)
    return out


def main(paths):
    print(json.dumps({p: parse(p) for p in paths}, indent=1))


if __name__ == "__main__":
    main(sys.argv[1:])

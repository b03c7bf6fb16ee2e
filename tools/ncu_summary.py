"""Summarise an ncu --set full report (read here, no GPU): key metrics + stall reasons."""
import csv
import io
import json
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "lts__t_sector_hit_rate.pct", "smsp__inst_executed.sum", "launch__occupancy_limit_registers",
        "l1tex__throughput.avg.pct_of_peak_sustained_active"]


def main(path, out_json=None):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    d = {}
    for i, h in enumerate(hdr):
        if h in KEYS:
            d[h] = (vals[i], units[i])
    stalls = sorted(((h.replace("smsp__pcsamp_warps_issue_stalled_", ""), float(vals[i] or 0))
                     for i, h in enumerate(hdr)
                     if h.startswith("smsp__pcsamp_warps_issue_stalled_")
                     and not h.endswith("not_issued")), key=lambda x: -x[1])
    for k in KEYS:
        if k in d:
            print(f"{k:60s} {d[k][0]:>16s} {d[k][1]}")
    tot = sum(v for _, v in stalls) or 1
    print("stall reasons (pc samples):", ", ".join(f"{n} {v / tot:.0%}" for n, v in stalls[:8]))
    if out_json:
        def num(k, scale=1.0):
            v, u = d[k]
            f = float(v.replace(",", ""))
            mult = {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "byte": 1, "us": 1e-6, "ms": 1e-3,
                    "ns": 1e-9}.get(u, 1.0)
            return f * mult
        traffic = num("dram__bytes_read.sum") + num("dram__bytes_write.sum")
        json.dump({"report": path, "dram_bytes_per_launch": traffic,
                   "dram_read_bytes": num("dram__bytes_read.sum"),
                   "dram_write_bytes": num("dram__bytes_write.sum"),
                   "duration_s": num("gpu__time_duration.sum"),
                   "dram_throughput_pct": float(d["gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"][0]),
                   "stalls": stalls[:8]}, open(out_json, "w"), indent=1)


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else None)

#!/usr/bin/env python
"""Summarise ncu artefacts for profiles/ (run here, no GPU needed).

  scripts/ncu_summary.py launches <launches.csv>      per-kernel share of device time
  scripts/ncu_summary.py full <prof.ncu-rep>          key counters of a --set full capture
  scripts/ncu_summary.py traffic <prof.ncu-rep> <key> <capture-name>
        record dram read + write bytes of the capture's (single) kernel launch in
        profiles/ncu_traffic.json under <key>, tagged with the library source
        hash (bench.py reports it only while the sources are unchanged)
"""
import csv
import io
import json
import os
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "l1tex__throughput.avg.pct_of_peak_sustained_active",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed",
    "l1tex__t_sector_hit_rate.pct", "lts__t_sector_hit_rate.pct",
    "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
    "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
    "l1tex__t_output_wavefronts_pipe_lsu_mem_global_op_ld.sum",
    "l1tex__t_sectors_pipe_lsu_mem_global_op_red.sum",
    "smsp__inst_executed.sum", "smsp__thread_inst_executed_per_inst_executed.ratio",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
    "launch__grid_size", "launch__block_size",
    "smsp__average_warp_latency_issue_stalled_long_scoreboard",
    "smsp__pcsamp_warps_issue_stalled_long_scoreboard",
]


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = None
    per = defaultdict(lambda: [0.0, 0])
    for r in rows:
        if "Kernel Name" in r and "Metric Value" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            if d.get("Metric Name") != "gpu__time_duration.sum":
                continue
            v = float(d["Metric Value"].replace(",", ""))
            unit = d.get("Metric Unit", "")
            scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3, "second": 1e6, "s": 1e6}.get(unit, 1.0)
            name = d["Kernel Name"].split("(")[0]
            per[name][0] += v * scale
            per[name][1] += 1
    tot = sum(v[0] for v in per.values()) or 1.0
    print(f"{'kernel':60s} {'launches':>8s} {'total us':>12s} {'share':>7s}")
    for k, (t, n) in sorted(per.items(), key=lambda kv: -kv[1][0]):
        print(f"{k[:60]:60s} {n:8d} {t:12.1f} {100 * t / tot:6.1f}%")


def full(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        print("kernel:", d.get("Kernel Name", "?")[:120])
        for k in KEYS:
            if k in d:
                print(f"  {k:70s} {d[k]:>20s} {units[hdr.index(k)]}")


def traffic(path, key, name):
    sys.path.insert(0, ROOT)
    import bench
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    d = dict(zip(hdr, rows[2]))
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
    tot = 0.0
    for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
        tot += float(d[k].replace(",", "")) * scale[units[hdr.index(k)]]
    tf = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        tj = json.load(open(tf))
    except Exception:   # noqa: BLE001
        tj = {}
    tj[key] = {"bytes": tot, "src_hash": bench.src_hash(), "capture": name,
               "kernel": d.get("Kernel Name", "?")[:80]}
    json.dump(tj, open(tf, "w"), indent=1, sort_keys=True)
    print(key, tot)


if __name__ == "__main__":
    cmd = sys.argv[1]
    if cmd == "traffic":
        traffic(sys.argv[2], sys.argv[3], sys.argv[4])
    else:
        {"launches": launches, "full": full}[cmd](sys.argv[2])

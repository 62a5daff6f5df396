#!/usr/bin/env python
"""Summarise ncu output for profiles/: a launch list (gpu__time_duration per
kernel, aggregated; shares of the step) and key metrics of `--set full` captures.

  python tools/ncu_summary.py launches gpurun_out/launches.csv > profiles/rN_launches.txt
  python tools/ncu_summary.py full gpurun_out/prof.ncu-rep > profiles/rN_ncu_<kernel>.txt
  python tools/ncu_summary.py traffic gpurun_out/traffic.csv   (-> profiles/traffic.json)
"""
import collections
import csv
import io
import subprocess
import sys

UNIT = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}

KEYS = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "smsp__inst_executed.sum", "lts__t_sectors_op_atom.sum", "lts__t_sectors_op_red.sum",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__throughput.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active"]


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr, data = None, []
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            data.append(dict(zip(hdr, r)))
    agg = collections.defaultdict(lambda: [0, 0.0])
    for d in data:
        if d["Metric Name"] != "gpu__time_duration.sum":
            continue
        v = float(d["Metric Value"].replace(",", "")) * UNIT.get(d["Metric Unit"], 1.0)
        k = d["Kernel Name"].split("(")[0]
        agg[k][0] += 1
        agg[k][1] += v
    tot = sum(v[1] for v in agg.values())
    print(f"# ncu launch list ({len(data)} launches, cold-cache, serialised): {path}")
    print(f"# {'total_us':>10} {'share':>6} {'n':>5} {'avg_us':>8}  kernel")
    for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"  {v[1]:10.1f} {100 * v[1] / tot:5.1f}% {v[0]:5d} {v[1] / v[0]:8.2f}  {k}")


def full(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    idx = {h: i for i, h in enumerate(hdr)}
    print(f"# ncu --set full: {path}")
    for r in rows[2:]:
        print("-" * 60)
        for k in KEYS:
            if k in idx:
                print(f"{k:62s} {r[idx[k]]} {units[idx[k]]}")


BYTES = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}


def traffic(path, out_json="profiles/traffic.json"):
    """Per-kernel DRAM traffic per launch (dram__bytes_read.sum + dram__bytes_write.sum,
    averaged over every captured launch) from an ncu --metrics CSV log; merged into
    profiles/traffic.json, which bench.py reports as roofline.traffic."""
    import json
    import os
    rows = list(csv.reader(open(path)))
    hdr, data = None, []
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            data.append(dict(zip(hdr, r)))
    per = collections.defaultdict(dict)
    for d in data:
        if d["Metric Name"] in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            v = float(d["Metric Value"].replace(",", "")) * BYTES.get(d["Metric Unit"], 1.0)
            per[(d["Kernel Name"].split("(")[0], d["ID"])][d["Metric Name"]] = v
    agg = collections.defaultdict(lambda: [0, 0.0])
    for (k, _), m in per.items():
        agg[k][0] += 1
        agg[k][1] += sum(m.values())
    cur = json.load(open(out_json)) if os.path.exists(out_json) else {}
    for k, (n, b) in agg.items():
        short = k.split("::")[-1].replace("_kernel", "")
        cur[short] = {"bytes_per_launch": b / n, "launches": n, "source": os.path.basename(path)}
        print(f"{short:24s} {n:6d} launches  {b / n:14.1f} B/launch")
    json.dump(cur, open(out_json, "w"), indent=1, sort_keys=True)


if __name__ == "__main__":
    {"launches": launches, "full": full, "traffic": traffic}[sys.argv[1]](sys.argv[2])

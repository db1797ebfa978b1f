#!/usr/bin/env python
"""Summarise ncu output: per-kernel launch shares from a launch-list CSV, and key
metrics + stall reasons per kernel from an --set full report.

usage: ncu_summary.py launches <launches.csv>
       ncu_summary.py report <file.ncu-rep> [--json out.json]
"""
import collections
import csv
import io
import json
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "lts__t_sector_hit_rate.pct", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "launch__shared_mem_per_block_dynamic", "launch__occupancy_limit_shared_mem"]


def _f(x):
    try:
        return float(str(x).replace(",", ""))
    except ValueError:
        return None


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = None
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            if d.get("Metric Name") != "gpu__time_duration.sum":
                continue
            k = d["Kernel Name"].split("(")[0]
            agg[k][0] += 1
            agg[k][1] += _f(d["Metric Value"]) or 0
    tot = sum(v[1] for v in agg.values()) or 1
    out = []
    for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
        out.append({"kernel": k, "launches": v[0], "total_us": v[1] / 1e3, "share": v[1] / tot})
        print(f"{k[:70]:70s} n={v[0]:5d} total={v[1] / 1e3:11.1f}us share={v[1] / tot:.3f}")
    return out


def report(path):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    res = []
    unit_of = dict(zip(hdr, units))
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
             "nsecond": 1e-3, "usecond": 1, "msecond": 1e3, "second": 1e6}
    for v in rows[2:]:
        d = dict(zip(hdr, v))
        name = d.get("Kernel Name", "?").split("(")[0]
        m = {}
        for k in KEYS:
            if k not in d:
                continue
            val, u = _f(d.get(k)), unit_of.get(k, "")
            if val is not None and u in scale:      # bytes in bytes, durations in microseconds
                val = val * scale[u]
                k = k + (".bytes" if "byte" in u else ".us")
            m[k] = val
        stalls = {h.replace("smsp__pcsamp_warps_issue_stalled_", ""): _f(d[h]) for h in hdr
                  if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("_not_issued")}
        stalls = dict(sorted(((k, v) for k, v in stalls.items() if v), key=lambda x: -x[1])[:8])
        res.append({"kernel": name, "metrics": m, "top_stalls": stalls})
        print(f"== {name}")
        for k, val in m.items():
            print(f"   {k:62s} {val}")
        print("   stalls:", stalls)
    return res


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        out = launches(sys.argv[2])
    else:
        out = report(sys.argv[2])
    if "--json" in sys.argv:
        with open(sys.argv[sys.argv.index("--json") + 1], "w") as f:
            json.dump(out, f, indent=1)

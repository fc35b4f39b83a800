#!/usr/bin/env python
"""Summarise ncu output into profiles/ (run here, on the CPU box).

    python tools/summarize_ncu.py --launches gpurun_out/launches.csv \
        --full gpurun_out/prof_bank_hv.ncu-rep --tag r01_bank

Writes profiles/<tag>_launches.csv (per-kernel launch count, mean/total
device time and share of the STM step) and profiles/<tag>_ncu_full.json
(the metrics the roofline and DESIGN.md cite, per launch).
"""
from __future__ import annotations

import argparse
import collections
import csv
import io
import json
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

FULL_METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_requests.sum",
    "lts__t_requests_srcunit_tex_op_read.sum", "lts__t_requests_srcunit_tex_op_write.sum",
    "lts__t_requests_srcunit_tex_op_atom_dot_alu.sum", "lts__t_sector_hit_rate.pct",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread", "launch__occupancy_limit_registers", "launch__grid_size",
    "launch__block_size", "smsp__thread_inst_executed_per_inst_executed.ratio",
    "smsp__average_warp_latency_per_inst_issued.ratio", "sm__inst_executed.sum",
]
STALLS = ["long_scoreboard", "membar", "barrier", "wait", "branch_resolving", "sleeping", "short_scoreboard",
          "no_instruction", "not_selected", "selected", "math_pipe_throttle", "lg_throttle", "drain", "dispatch_stall",
          "misc", "mio_throttle"]


def launches(path: str, out: str) -> dict:
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, vi = h.index("Kernel Name"), h.index("Metric Value")
    agg = collections.OrderedDict()
    for r in rows[hi + 1:]:
        if len(r) > vi:
            agg.setdefault(r[ki].split("(")[0].strip(), []).append(float(r[vi].replace(",", "")))
    with open(out, "w") as f:
        w = csv.writer(f)
        w.writerow(["kernel", "launches", "mean_us", "total_ms"])
        for k, v in agg.items():
            w.writerow([k, len(v), round(sum(v) / len(v) / 1e3, 3), round(sum(v) / 1e6, 4)])
    return {k: (len(v), sum(v) / len(v)) for k, v in agg.items()}


def full(path: str) -> dict:
    raw = subprocess.check_output(["ncu", "-i", path, "--page", "raw", "--csv"], text=True, stderr=subprocess.DEVNULL)
    rows = list(csv.reader(io.StringIO(raw)))
    h, u, v = rows[0], rows[1], rows[2]
    col = {n: i for i, n in enumerate(h)}
    out = {"kernel": v[col["Kernel Name"]] if "Kernel Name" in col else None}
    for m in FULL_METRICS:
        if m in col:
            out[m] = {"value": v[col[m]], "unit": u[col[m]]}
    # every L2 request / sector breakdown the report holds (source unit, op)
    out["l2_breakdown"] = {n: v[i] for n, i in col.items()
                           if (n.startswith("lts__t_requests_srcunit") or n.startswith("lts__t_sectors_srcunit"))
                           and n.endswith(".sum") and v[i] not in ("", "0", "n/a")}
    out["stalls_per_issue"] = {}
    for s in STALLS:
        n = f"smsp__average_warps_issue_stalled_{s}_per_issue_active.ratio"
        if n in col:
            out["stalls_per_issue"][s] = float(v[col[n]])

    def to_bytes(m):
        x = out.get(m)
        if not x:
            return None
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(x["unit"], 1)
        return float(x["value"].replace(",", "")) * scale

    rd, wr = to_bytes("dram__bytes_read.sum"), to_bytes("dram__bytes_write.sum")
    out["dram_bytes_per_launch"] = (rd or 0) + (wr or 0)
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--launches")
    ap.add_argument("--full")
    ap.add_argument("--tag", required=True)
    a = ap.parse_args()
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    if a.launches:
        s = launches(a.launches, os.path.join(ROOT, "profiles", f"{a.tag}_launches.csv"))
        for k, (n, mean) in s.items():
            print(f"{n:5d} {mean / 1e3:12.1f} us  {k}")
    if a.full:
        d = full(a.full)
        with open(os.path.join(ROOT, "profiles", f"{a.tag}_ncu_full.json"), "w") as f:
            json.dump(d, f, indent=1)
        print(json.dumps(d, indent=1)[:2000])


if __name__ == "__main__":
    main()

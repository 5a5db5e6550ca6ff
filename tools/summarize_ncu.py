#!/usr/bin/env python
"""Summarize ncu reports / launch lists into profiles/ (committed evidence).

  python tools/summarize_ncu.py full  <report.ncu-rep> <out.md> [traffic_key]
  python tools/summarize_ncu.py launches <launches.csv> <out.md>

`full` prints per-kernel key metrics (duration, DRAM bytes, throughputs, stall
reasons) and, with traffic_key, records dram read+write bytes per launch into
profiles/traffic.json (bench.py reports it as roofline.traffic).
"""
import collections
import csv
import io
import json
import os
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sectors.sum",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__throughput.avg.pct_of_peak_sustained_active",
    "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__grid_size", "launch__block_size", "launch__registers_per_thread",
    "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem", "smsp__inst_executed.sum",
    "l1tex__m_l1tex2xbar_req_cycles_active.avg.pct_of_peak_sustained_elapsed", "l1tex__t_sector_hit_rate.pct",
    "lts__t_sector_hit_rate.pct", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
]


def to_bytes(val, unit):
    v = float(val.replace(",", ""))
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}.get(unit, 1)
    return v * mult


def full(rep, out, key=None):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, units = rows[0], rows[1]
    lines = [f"# ncu --set full summary: `{os.path.basename(rep)}`", ""]
    traffic = []
    for r in rows[2:]:
        name = r[h.index("Kernel Name")]
        lines.append(f"## {name}")
        lines.append("")
        lines.append("| metric | value | unit |")
        lines.append("|---|---|---|")
        for k in KEYS:
            if k in h:
                i = h.index(k)
                lines.append(f"| {k} | {r[i]} | {units[i]} |")
        stalls = []
        for i, k in enumerate(h):
            if k.startswith("smsp__average_warps_issue_stalled") and not k.endswith("not_issued"):
                try:
                    v = float(r[i])
                except ValueError:
                    continue
                if v >= 0.5:
                    stalls.append((v, k.replace("smsp__average_warps_issue_stalled_", "").replace(
                        "_per_issue_active.ratio", "")))
        stalls.sort(reverse=True)
        lines.append("")
        lines.append("stall reasons (warps per issue): " + ", ".join(f"{n} {v:.2f}" for v, n in stalls[:8]))
        lines.append("")
        rd = to_bytes(r[h.index("dram__bytes_read.sum")], units[h.index("dram__bytes_read.sum")])
        wr = to_bytes(r[h.index("dram__bytes_write.sum")], units[h.index("dram__bytes_write.sum")])
        if key and key.split("@")[0] in name:
            traffic.append(rd + wr)
    open(out, "w").write("\n".join(lines) + "\n")
    if key and traffic:
        p = os.path.join(os.path.dirname(out), "traffic.json")
        d = json.load(open(p)) if os.path.exists(p) else {}
        d[key] = int(sum(traffic) / len(traffic))
        json.dump(d, open(p, "w"), indent=1, sort_keys=True)
    print(out)


def launches(csvf, out):
    rows = list(csv.reader(open(csvf)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = collections.OrderedDict()
    for r in rows[hi + 1:]:
        if len(r) > vi:
            agg.setdefault(r[ki], []).append(float(r[vi].replace(",", "")))
    tot = sum(sum(v) for v in agg.values())
    lines = [f"# ncu launch list (gpu__time_duration.sum, --clock-control none): `{os.path.basename(csvf)}`", "",
             "Cold-cache, serialized launches: compare SHARES, not absolute times.", "",
             "| kernel | launches | mean | total | share |", "|---|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        lines.append(f"| `{k[:90]}` | {len(v)} | {sum(v) / len(v):.1f} | {sum(v):.1f} | {sum(v) / tot:.3f} |")
    open(out, "w").write("\n".join(lines) + "\n")
    print(out)


if __name__ == "__main__":
    if sys.argv[1] == "full":
        full(sys.argv[2], sys.argv[3], sys.argv[4] if len(sys.argv) > 4 else None)
    else:
        launches(sys.argv[2], sys.argv[3])

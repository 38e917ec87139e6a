#!/usr/bin/env python3
"""Summarise ncu captures (.ncu-rep --set full) and launch lists for profiles/.

    python scripts/ncu_summary.py rep REP.ncu-rep [--key n16_b1048576_c32] [--traffic-json profiles/ncu_traffic.json]
    python scripts/ncu_summary.py launches LAUNCHES.csv
"""
import csv
import io
import json
import subprocess
import sys
from collections import defaultdict

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("dram__cycles_active.avg.pct_of_peak_sustained_elapsed", "DRAM active % of peak"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__shared_mem_per_block_dynamic", "dyn smem/block"),
    ("launch__occupancy_limit_registers", "occupancy limit (regs)"),
    ("launch__occupancy_limit_shared_mem", "occupancy limit (smem)"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active %"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "FMA pipe %"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "LSU pipe %"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smem wavefronts"),
    ("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "global ld sectors"),
    ("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "global ld requests"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("sm__cycles_elapsed.avg.per_second", "SM clock"),
]
STALLS = ["no_instruction", "long_scoreboard", "short_scoreboard", "wait", "mio_throttle",
          "lg_throttle", "math_pipe_throttle", "barrier", "branch_resolving", "misc", "selected",
          "not_selected", "dispatch_stall", "sleeping", "drain", "membar", "tex_throttle"]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    return [(dict(zip(hdr, r)), dict(zip(hdr, units))) for r in rows[2:]]


def rep_summary(rep, key=None, traffic_json=None):
    lines = []
    for vals, units in raw(rep):
        name = vals.get("Kernel Name", "?")
        lines.append(f"### {name}\n")
        lines.append("| metric | value |\n|---|---|")
        for m, label in METRICS:
            if m in vals:
                lines.append(f"| {label} (`{m}`) | {vals[m]} {units.get(m, '')} |")
        st = []
        for s in STALLS:
            m = f"smsp__average_warps_issue_stalled_{s}_per_issue_active.ratio"
            if m in vals and vals[m] not in ("", "n/a"):
                st.append((float(vals[m]), s))
        st.sort(reverse=True)
        lines.append("| stalls per issued instruction (top) | " +
                     ", ".join(f"{s} {v:.2f}" for v, s in st[:6]) + " |")
        rd = float(vals.get("dram__bytes_read.sum", "0") or 0)
        wr = float(vals.get("dram__bytes_write.sum", "0") or 0)
        ur, uw = units.get("dram__bytes_read.sum", ""), units.get("dram__bytes_write.sum", "")
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
        tot = rd * scale.get(ur, 1) + wr * scale.get(uw, 1)
        lines.append(f"| DRAM read+write bytes per launch | {tot:.4g} B |\n")
        if key and traffic_json:
            try:
                d = json.load(open(traffic_json))
            except FileNotFoundError:
                d = {}
            d[key] = {"dram_bytes_per_launch": tot, "kernel": name, "source": rep}
            json.dump(d, open(traffic_json, "w"), indent=1)
    return "\n".join(lines)


def launches(path):
    rows = list(csv.DictReader(l for l in open(path) if not l.startswith("==")))
    agg = defaultdict(list)
    for r in rows:
        if r.get("Metric Name") == "gpu__time_duration.sum":
            agg[r["Kernel Name"]].append(float(r["Metric Value"]))
    tot = sum(sum(v) for v in agg.values())
    out = ["| kernel | launches | mean ns | share of GPU time |", "|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        out.append(f"| `{k[:90]}` | {len(v)} | {sum(v) / len(v):.0f} | {100 * sum(v) / tot:.1f}% |")
    return "\n".join(out)


if __name__ == "__main__":
    if sys.argv[1] == "rep":
        key = tj = None
        if "--key" in sys.argv:
            key = sys.argv[sys.argv.index("--key") + 1]
        if "--traffic-json" in sys.argv:
            tj = sys.argv[sys.argv.index("--traffic-json") + 1]
        print(rep_summary(sys.argv[2], key, tj))
    else:
        print(launches(sys.argv[2]))

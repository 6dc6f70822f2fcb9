#!/usr/bin/env python
"""Summarise ncu outputs for profiles/:

    python tools/ncu_summary.py launches <launches.csv>          # per-kernel share of the launch list
    python tools/ncu_summary.py report <prof.ncu-rep> [...]      # key counters of a --set full capture
"""
from __future__ import annotations

import csv
import io
import re
import subprocess
import sys
from collections import defaultdict

KEYS = [
    ("gpu__time_duration.sum", "duration (ns)"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__occupancy_limit_shared_mem", "occupancy limit (smem, CTAs/SM)"),
    ("sm__warps_active.avg.per_cycle_active", "warps active / SM"),
    ("sm__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", "ALU pipe % (inst executed)"),
    ("sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "ALU pipe cycles active %"),
    ("sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_elapsed", "FMA-heavy pipe cycles %"),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "FMA pipe cycles %"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "LSU pipe %"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed", "smem wavefronts %"),
    ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "smem load bank conflicts"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("lts__t_bytes.sum", "L2 bytes"),
    ("smsp__inst_executed.sum", "warp instructions"),
]
STALLS = re.compile(r"smsp__average_warps_issue_stalled_(\w+)_per_issue_active\.ratio")


def short_name(k: str) -> str:
    k = k.replace("<unnamed>", "anon").replace("(anonymous namespace)", "anon")
    k = re.sub(r"\(.*$", "", k)           # drop the argument list
    k = re.sub(r"<[^<>]*>", "", k)        # drop template args
    return k.split("::")[-1].strip()


def launches(path):
    text = open(path).read()
    lines = text.splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    rows = list(csv.DictReader(io.StringIO("\n".join(lines[start:]))))
    agg = defaultdict(float)
    cnt = defaultdict(int)
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(r["Metric Value"].replace(",", ""))
        scale = {"ns": 1.0, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6, "nsecond": 1.0}.get(r["Metric Unit"], 1.0)
        name = short_name(r["Kernel Name"])
        agg[name] += v * scale
        cnt[name] += 1
    tot = sum(agg.values())
    out = [f"launch list: {path} ({sum(cnt.values())} launches, {tot / 1e6:.3f} ms serialised, cold-cache)",
           "", "| kernel | launches | total ms | share |", "|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda x: -x[1]):
        out.append(f"| {k} | {cnt[k]} | {v / 1e6:.3f} | {100 * v / tot:.1f}% |")
    return "\n".join(out)


def report(path):
    """path: a .ncu-rep, or the `ncu -i <rep> --page raw --csv` export of one (.raw.csv)."""
    if path.endswith(".csv"):
        raw = open(path).read()
    else:
        raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    out = []
    for vals in rows[2:]:
        d = dict(zip(hdr, vals))
        u = dict(zip(hdr, units))
        out.append(f"### {short_name(d.get('Kernel Name', '?'))}  ({path})")
        out.append("")
        out.append("| counter | value |")
        out.append("|---|---|")
        for k, label in KEYS:
            if k in d:
                out.append(f"| {label} (`{k}`) | {d[k]} {u.get(k, '')} |")
        stalls = sorted(((STALLS.match(k).group(1), float(v or 0)) for k, v in d.items() if STALLS.match(k)),
                        key=lambda x: -x[1])
        out.append("| top stalls (warps per issue) | " + ", ".join(f"{n} {v:.2f}" for n, v in stalls[:7]) + " |")
        out.append("")
    return "\n".join(out)


if __name__ == "__main__":
    mode = sys.argv[1]
    if mode == "launches":
        print(launches(sys.argv[2]))
    else:
        for p in sys.argv[2:]:
            print(report(p))

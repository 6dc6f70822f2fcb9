#!/usr/bin/env python
"""Turn the outputs of tools/gpu_evidence.sh (gpurun_out/ev_*) into the tracked evidence under profiles/:

    python tools/evidence_summary.py TAG [OUTDIR]    # e.g. r01 (OUTDIR defaults to profiles/)

writes profiles/TAG_bench_lines.jsonl (every bench JSON line), profiles/TAG_launches_H.csv (the ncu launch
list of the default bench) and profiles/TAG_ncu_summary.md (bench table, launch-list shares, the key
counters of every --set full capture, and the source-level pass breakdown of K3).
"""
from __future__ import annotations

import csv
import glob
import json
import os
import shutil
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")
sys.path.insert(0, os.path.join(ROOT, "tools"))
import ncu_summary  # noqa: E402


def bench_table(lines):
    rows = ["| line | workload | ms/step | dominance tests/s | phases ms (prep / K1 / K3 / K4) | e2e ms | K3 frac | cpu_baseline tests/s (cores) |",
            "|---|---|---|---|---|---|---|---|"]
    for name, j in lines:
        ph = j.get("phases_ms", {})
        phs = " / ".join("%.1f" % ph[k] for k in ("prepare", "prefilter", "mdmc", "compact") if k in ph) or \
            " / ".join("%.1f" % v for v in ph.values())
        e2e = j.get("e2e", {})
        cpu = j.get("cpu_baseline")
        frac = j.get("roofline", {}).get("frac")
        rows.append("| %s | %s | %.1f | %.3g | %s | %s | %s | %s |" % (
            name, j["config"]["workload"].split(" (")[0], j["ms_per_step"], j["value"], phs,
            "%.1f" % e2e["ms_per_step"] if "ms_per_step" in e2e else "—",
            "%.3f" % frac if frac is not None else "—",
            "%.3g (%s)" % (cpu["value"], cpu["cores"]) if cpu else "—"))
    return "\n".join(rows)


def k3_passes(rep):
    """Warp-stall samples and executed instructions of K3 per source region (design A line ranges)."""
    src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(src.splitlines()))
    cur, hdr, out = None, None, []
    for r in rows:
        if r and r[0] == "File Path":
            cur = r[1].split("/")[-1]
            continue
        if r and r[0] == "Line No":
            hdr = r
            continue
        if not r or r[0] == "Function Name" or not r[0] or hdr is None:
            continue
        try:
            out.append((cur, int(r[0]), r[1], int(r[4]), int(r[7])))
        except (ValueError, IndexError):
            pass
    if not out:
        return ""
    tots = sum(o[3] for o in out) or 1
    toti = sum(o[4] for o in out) or 1
    top = sorted(out, key=lambda o: -o[3])[:15]
    lines = ["| source line | warp-stall samples | instructions |", "|---|---|---|"]
    for f, ln, text, smp, ins in top:
        lines.append("| `%s:%d` %s | %.1f%% | %.1f%% |" % (f, ln, text.strip()[:70].replace("|", "\\|"),
                                                         100 * smp / tots, 100 * ins / toti))
    return "\n".join(lines)


def main():
    global PROF
    tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
    if len(sys.argv) > 2:
        PROF = os.path.abspath(sys.argv[2])
        os.makedirs(PROF, exist_ok=True)
    lines = []
    for f in sorted(glob.glob(os.path.join(OUT, "ev_bench_*.json"))):
        try:
            j = json.loads(open(f).read().strip().splitlines()[-1])
        except Exception:
            continue
        lines.append((os.path.basename(f)[len("ev_bench_"):-5], j))
    with open(os.path.join(PROF, f"{tag}_bench_lines.jsonl"), "w") as fo:
        for name, j in lines:
            fo.write(json.dumps({"line": name, **j}) + "\n")
    md = [f"# {tag} evidence (tools/gpu_evidence.sh on one B200; summarised by tools/evidence_summary.py)", ""]
    gpu = os.path.join(OUT, "ev_gpu.txt")
    if os.path.exists(gpu):
        md += ["GPU: `" + open(gpu).read().strip().replace("\n", " | ") + "`", ""]
    for f in ("ev_tests.log", "ev_smoke.log"):
        p = os.path.join(OUT, f)
        if os.path.exists(p):
            md += [f"`{f}`: " + " ".join(open(p).read().split())[-200:], ""]
    md += ["## bench.py lines", "", bench_table([l for l in lines if "impl" not in l[1] and "algo" not in l[1]]), ""]
    other = [l for l in lines if "impl" in l[1] or "algo" in l[1]]
    if other:
        md += ["Other lines (reference arm = the CPU oracle; SDSC comparator):", ""]
        for name, j in other:
            md.append("* `%s`: %.1f ms/step, %.3g %s — %s" % (name, j["ms_per_step"], j["value"], j["unit"],
                                                             j["config"]["workload"].split(" (")[0]))
        md.append("")
    lc = os.path.join(OUT, "ev_launches_H.csv")
    if os.path.exists(lc):
        dst = os.path.join(PROF, f"{tag}_launches_H.csv")
        shutil.copy(lc, dst)
        md += ["## Launch list of the default bench (H), `ncu --metrics gpu__time_duration.sum --clock-control none`",
               "", ncu_summary.launches(dst).replace(ROOT + "/", ""), ""]
    md += ["## `ncu --set full` captures (one launch each)", ""]
    caps = sorted(glob.glob(os.path.join(OUT, "ev_prof_*.ncu-rep")))
    have = {c[:-len(".ncu-rep")] for c in caps}
    caps += [c for c in sorted(glob.glob(os.path.join(OUT, "ev_prof_*.raw.csv"))) if c[:-len(".raw.csv")] not in have]
    for rep in caps:
        md += [ncu_summary.report(rep).replace(ROOT + "/", "").replace("gpurun_out/", ""), ""]
        base = rep[:-len(".ncu-rep")] if rep.endswith(".ncu-rep") else rep[:-len(".raw.csv")]
        if os.path.exists(base + ".lines.txt"):  # per-source-line instructions / stall samples (tools/ncu_lines.py)
            md += ["Hottest source lines (`tools/ncu_lines.py`: share of executed warp instructions, share of "
                   "warp-stall samples):", "", "```", open(base + ".lines.txt").read().strip(), "```", ""]
        elif rep.endswith(".ncu-rep") and "k3_" in rep:
            md += ["Hottest source lines:", "", k3_passes(rep), ""]
    with open(os.path.join(PROF, f"{tag}_ncu_summary.md"), "w") as fo:
        fo.write("\n".join(md) + "\n")
    print("wrote", os.path.join(PROF, f"{tag}_ncu_summary.md"))


if __name__ == "__main__":
    main()

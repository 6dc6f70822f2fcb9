"""One-line summaries of bench.py JSON lines: python tools/bench_summary.py FILE [LABEL] (or stdin)."""
import json
import sys

src = open(sys.argv[1]) if len(sys.argv) > 1 else sys.stdin
label = sys.argv[2] if len(sys.argv) > 2 else ""
for line in src:
    line = line.strip()
    if not line.startswith("{"):
        continue
    d = json.loads(line)
    w = d.get("work_per_step", {})
    print(label, d["config"]["workload"].split(" (")[0], "ms=%.1f" % d["ms_per_step"],
          {k: round(v, 1) for k, v in d["phases_ms"].items()}, "frac=%.3f" % d["roofline"]["frac"],
          "n_ext=%d" % d["config"]["n_ext"], {k: "%.3g" % v for k, v in w.items()})

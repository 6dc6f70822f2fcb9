"""One-line summaries of bench.py JSON lines (stdin)."""
import json
import sys

for line in sys.stdin:
    line = line.strip()
    if not line.startswith("{"):
        continue
    d = json.loads(line)
    w = d.get("work_per_step", {})
    print(d["config"]["workload"].split(" (")[0], "ms=%.1f" % d["ms_per_step"],
          {k: round(v, 1) for k, v in d["phases_ms"].items()}, "frac=%.3f" % d["roofline"]["frac"],
          "n_ext=%d" % d["config"]["n_ext"],
          "skip=%.3f" % (1 - w.get("k3_pair", 0) / max(1, 32 * w.get("k3_box", 1))),
          "k3_miss=%.3g" % w.get("k3_miss", 0), "k1_skip=%.3f" % (1 - w.get("k1_pair", 0) / max(1, 32 * w.get("k1_box", 1))))

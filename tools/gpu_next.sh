#!/bin/bash
# GPU-box helper: NEXT-1 / NEXT-2 evidence at d = 16 (C4): the lattice, the HashCube output (w = 32) and the
# partial skycube at d' = 2, 4, 8, 12 -- device build and e2e (C-ABI, host buffers) with the bytes copied D2H.
mkdir -p gpurun_out
for v in "lattice 0" "hashcube 0" "lattice 2" "lattice 4" "lattice 8" "lattice 12"; do
  set -- $v
  timeout 900 python bench.py --steps 3 --warmup 2 --config ${CFG:-C4} --no-cpu --output $1 --max-level $2 \
    2>/dev/null | tail -1 > gpurun_out/r02_next_${CFG:-C4}_$1_$2.json
  python - "$1" "$2" <<'PY'
import json, sys
try:
    d = json.load(open(f"gpurun_out/r02_next_C4_{sys.argv[1]}_{sys.argv[2]}.json"))
    e = d.get("e2e", {})
    print(sys.argv[1], "max_level", sys.argv[2], "device ms %.1f" % d["ms_per_step"], "e2e ms %.1f" % e.get("ms_per_step", -1),
          "d2h GB %.2f" % (e.get("d2h_bytes_per_step", 0) / 1e9), d["config"]["output"], "ids", d["config"].get("total_ids"))
except Exception as ex:
    print("failed", sys.argv, ex)
PY
done

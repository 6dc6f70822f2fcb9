#!/usr/bin/env python
"""K3 time on a custom workload through the C-ABI (skycube_build_ex stats, median of REPS builds):

    python tools/k3_time.py DIST N D SEED [REPS]      # e.g. A 500000 14 9

SKYCUBE_LIB / SKYCUBE_K3_* select the library and tuning overrides (tools/gpu_*ab.sh).  A design tool for
A/B runs at dimensionalities outside BASELINE.json's configs; not a bench line."""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import datagen  # noqa: E402
import paper_conf_sigmod_boghcsa17_b200 as sky  # noqa: E402

dist, n, d, seed = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
reps = int(sys.argv[5]) if len(sys.argv) > 5 else 3
x = datagen.generate(dist, n, d, seed)
ms = []
for _ in range(reps + 1):
    with sky.skycube_build_raw(x, lists=False, stats=True) as r:
        ms.append(r.stats["ms_mdmc"])
        n_ext = r.n_ext
print(json.dumps({"workload": f"{dist} n={n} d={d} seed={seed}", "lib": os.path.basename(os.environ.get("SKYCUBE_LIB", "libskycube.so")),
                  "design": os.environ.get("SKYCUBE_K3_DESIGN", "auto"), "n_ext": n_ext, "k3_ms": float(np.median(ms[1:]))}))

"""GPU debugging aid: for mismatching rows, count bits the GPU sets that the oracle does not (+) and vice versa."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import datagen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_sigmod_boghcsa17_b200 as sky  # noqa: E402

for dist, n, d, seed in [("A", 2500, 13, 6), ("A", 2500, 14, 6), ("I", 2500, 13, 6)]:
    x = datagen.generate(dist, n, d, seed)
    want = oracle.rows_b(x)
    for rep in range(int(os.environ.get("REPS", "6"))):
        r = sky.skycube_build(x)
        got = r["rows"]
        bad = np.nonzero((got != want).any(axis=1))[0]
        extra = sum(int(np.unpackbits((got[b] & ~want[b]).view(np.uint8)).sum()) for b in bad)
        missing = sum(int(np.unpackbits((want[b] & ~got[b]).view(np.uint8)).sum()) for b in bad)
        print(dist, n, d, "rep", rep, "bad", bad.size, "gpu-only bits", extra, "oracle-only bits", missing,
              bad[:3].tolist(), flush=True)

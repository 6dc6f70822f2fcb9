"""GPU debugging aid: mismatch counts of the CUDA path vs Oracle B over (dist, n, d, mode, ext) cases."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import datagen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_sigmod_boghcsa17_b200 as sky  # noqa: E402

cases = [("A", 2500, 13, 6), ("A", 1000, 13, 6), ("A", 2500, 12, 6), ("A", 2500, 14, 6), ("A", 2500, 16, 6),
         ("I", 2500, 13, 6), ("A", 2500, 11, 6)]
for dist, n, d, seed in cases:
    x = datagen.generate(dist, n, d, seed)
    want = oracle.rows_b(x)
    for mode in ["", "0", "1", "2"]:
        for ext in [False, True]:
            os.environ["SKYCUBE_K3_MODE"] = mode
            r = sky.skycube_build(x, ext_membership=ext)
            bad = np.nonzero((r["rows"] != want).any(axis=1))[0]
            print(dist, n, d, "mode", mode or "auto", "ext", ext, "bad rows", bad.size, bad[:4], flush=True)

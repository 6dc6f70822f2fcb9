"""Debug helper: GlobalTie (mode 0) vs oracle at d = 16 on tie-heavy data; prints the differing bits."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import datagen, oracle
import paper_conf_sigmod_boghcsa17_b200 as sky
x = datagen.small_int_grid(433, 16, 3, 4242)
want = oracle.rows_b(x)
for mode in (1, 0, 0):
    sky.set_tuning("k3_mode", mode)
    r = sky.skycube_build(x)
    bad = np.nonzero((r["rows"] != want).any(axis=1))[0]
    print("mode", mode, "bad rows", bad.size, bad[:8])
    for p in bad[:3]:
        g, w = r["rows"][p], want[p]
        extra = sum(bin(int(a) & ~int(b) & 0xffffffff).count("1") for a, b in zip(g, w))
        missing = sum(bin(int(b) & ~int(a) & 0xffffffff).count("1") for a, b in zip(g, w))
        print("  p", p, "extra member bits", extra, "missing member bits", missing)

#!/usr/bin/env python
"""One pipeline build of a synthetic workload, for ncu captures of a kernel at a size other than a BASELINE
config (e.g. d = 16 at 300K points: the full C4 footprint makes ncu's replay save/restore fail):
    python tools/prof_run.py DIST N D SEED [--hashcube W] [--max-level L]"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import datagen  # noqa: E402
from paper_conf_sigmod_boghcsa17_b200.pipeline import DeviceSkycube  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("dist")
ap.add_argument("n", type=int)
ap.add_argument("d", type=int)
ap.add_argument("seed", type=int)
ap.add_argument("--hashcube", type=int, default=0)
ap.add_argument("--max-level", type=int, default=0)
a = ap.parse_args()
x = datagen.generate(a.dist, a.n, a.d, a.seed)
eng = DeviceSkycube(0)
out = eng.build(torch.from_numpy(x).cuda(), lists=not a.hashcube, membership=True, hashcube_w=a.hashcube,
                max_level=a.max_level)
torch.cuda.synchronize()
print({"n_ext": out["n_ext"], "counters": eng.ctx.counters()})

#!/usr/bin/env python
"""Per-rank device work of an N-GPU run, measured on one GPU with CUDA events: for every rank r of WORLD, the
sharded prepare (K0 + K2 on its slice of the dimensions, pipeline.dim_slice; then the replicated finish), the
K1 blocks it processes (pipeline.prefilter_assignment: b = r mod WORLD) and its contiguous K3 task range
(pipeline.task_range), run one rank after the other on the same device.  The slowest rank is the critical
path of the sharded build; the collectives are small (the codes all-gather, n x d x 2 bytes;
n bytes of S+ flags; WORLD x 2^d counts).

    python tools/k3_shard_time.py CONFIG WORLD [REPS]      # e.g. H 8

A design tool for the multi-GPU projection; not a bench line."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import datagen  # noqa: E402
from paper_conf_sigmod_boghcsa17_b200 import Context  # noqa: E402
from paper_conf_sigmod_boghcsa17_b200.pipeline import dim_slice, prefilter_assignment, rows_buffer_words, task_range  # noqa: E402

cfg, world = sys.argv[1], int(sys.argv[2])
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
x = datagen.config(cfg).data()
n, d = x.shape
pts = torch.from_numpy(x).cuda()
ctx = Context(0)
sp = torch.cuda.current_stream().cuda_stream


def timed(fn):
    ms = []
    for _ in range(reps + 1):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ms.append(a.elapsed_time(b))
    ms = sorted(ms[1:])
    return ms[len(ms) // 2]


# sharded prepare: K0 + K2 on each rank's slice of the dimensions, then the replicated finish
per = -(-d // world)
codes = torch.zeros((world * per, n), dtype=torch.int16, device="cuda")
R32 = torch.zeros(d, dtype=torch.int32, device="cuda")
mo32 = torch.zeros(d, dtype=torch.int32, device="cuda")
prep = []
for r in range(world):
    b, e = dim_slice(d, world, r)
    prep.append(timed(lambda: ctx.prepare_dims(pts.data_ptr(), n, d, b, e, codes[r * per:].data_ptr(), R32.data_ptr(),
                                               mo32.data_ptr(), sp)))
dm = torch.cat([codes[r * per: r * per + (dim_slice(d, world, r)[1] - dim_slice(d, world, r)[0])]
                for r in range(world)]).contiguous()
fin = timed(lambda: ctx.prepare_finish(dm.data_ptr(), R32.data_ptr(), mo32.data_ptr(), sp))
full = timed(lambda: ctx.prepare(pts.data_ptr(), n, d, sp))
ext8 = torch.zeros(n, dtype=torch.uint8, device="cuda")
k1 = []
for r in range(world):
    off, step = prefilter_assignment(r, world)
    k1.append(timed(lambda: ctx.prefilter(ext8.data_ptr(), off, step, sp)))
ctx.prefilter(ext8.data_ptr(), 0, 1, sp)
m = ctx.set_ext(ext8.data_ptr(), sp)
rows = torch.empty(rows_buffer_words(m, d), dtype=torch.int32, device="cuda")
k3 = []
for r in range(world):
    j0, j1 = task_range(m, world, r)
    k3.append(timed(lambda: ctx.mdmc(rows.data_ptr(), j0, j1, 0, sp)))
print(json.dumps({"config": cfg, "world": world, "lib": os.path.basename(os.environ.get("SKYCUBE_LIB", "libskycube.so")),
                  "prepare_ms_one_gpu": full, "prepare_dims_ms_per_rank": [round(v, 3) for v in prep],
                  "prepare_finish_ms": fin, "prepare_ms_max": max(prep) + fin,
                  "k1_ms_per_rank": [round(v, 3) for v in k1], "k3_ms_per_rank": [round(v, 3) for v in k3],
                  "k1_ms_max": max(k1), "k3_ms_max": max(k3)}))

"""Offline full-size Oracle B digests — TEST INFRASTRUCTURE (calls only ``oracle/`` and ``datagen``).

For a BASELINE config (H, C3A, C5, C4 …) this runs Oracle B (``oracle.rows_b``: per point p against
every q of P, then superset closures — Def. 1-3) over EVERY point of the
synthetic workload, plus ``oracle.ext_full`` (S+(P), Alg. 3 line 2, L320) and ``oracle.lattice``
(Fig. 1a), and writes SHA-256 digests of the whole output to
``tests/golden/fullsize_digests.json``:

* ``rows``      — sha256 of membership rows ``uint32[n][W]`` (little endian, id order),
* ``row_blocks`` — sha256 of every block of ``BLOCK`` consecutive rows (localises a mismatch),
* ``ext_ids``   — sha256 of ``int32`` ascending ids of S+(P), and ``n_ext``,
* ``offsets``   — sha256 of the lattice offsets ``int64[2^d+1]`` (and the offsets themselves for d ≤ 12),
* ``ids``       — sha256 of the lattice ids ``int32[offsets[-1]]``,
* ``data``      — sha256 of the float32 input (so a generator drift is caught before the comparison).

Nothing here comes from the CUDA path.  The GPU test ``tests/test_gpu_digest.py`` hashes the GPU
output built through the bench launch path and compares it with these values.

The run is chunked and resumable (Oracle B on H takes about 2 h on 8 cores): every chunk of
``CHUNK`` points is stored under ``.oracle_work/<cfg>/`` (git-ignored; ``SKYCUBE_ORACLE_WORK`` moves it, e.g.
out of the tree for C4's 8 GB of rows) and skipped when present.  The wall and CPU time of every chunk is
recorded, so the file also holds a full-size, un-extrapolated Oracle B timing on this host.

Usage: ``OMP_NUM_THREADS=8 nice -n 19 python tools/oracle_digest.py H C3A C5 [C4]``
"""
from __future__ import annotations

import argparse
import hashlib
import json
import os
import platform
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import datagen  # noqa: E402
import oracle   # noqa: E402

GOLDEN = os.path.join(ROOT, "tests", "golden", "fullsize_digests.json")
WORK = os.environ.get("SKYCUBE_ORACLE_WORK") or os.path.join(ROOT, ".oracle_work")
CHUNK = 8192
BLOCK = 4096


def sha(a: np.ndarray) -> str:
    # hashes the array's buffer in place (C4's 28 GB lattice must not be copied)
    return hashlib.sha256(memoryview(np.ascontiguousarray(a)).cast("B")).hexdigest()


def file_sha(path: str) -> str:
    return hashlib.sha256(open(path, "rb").read()).hexdigest()


def cpu_model() -> str:
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True).stdout
        for line in out.splitlines():
            if line.startswith("Model name:"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return platform.processor()


def load_golden() -> dict:
    if os.path.exists(GOLDEN):
        return json.load(open(GOLDEN))
    return {"_about": ("Full-size Oracle B digests written by tools/oracle_digest.py (calls only oracle/ "
                       "and datagen). Row r of 'rows' is point id r; bit delta of word delta>>5 <=> "
                       "p in S_delta(P) (Def. 3, PAPER.md L110)."),
            "configs": {}}


def save_golden(g: dict) -> None:
    tmp = GOLDEN + ".tmp"
    with open(tmp, "w") as f:
        json.dump(g, f, indent=1, sort_keys=True)
        f.write("\n")
    os.replace(tmp, GOLDEN)


def run(name: str, chunk: int) -> dict:
    cfg = datagen.config(name)
    x = cfg.data()
    n, d = x.shape
    W = oracle.words_per_row(d)
    wdir = os.path.join(WORK, name)
    os.makedirs(wdir, exist_ok=True)
    threads = oracle.num_threads()
    timing_path = os.path.join(wdir, "timing.json")
    timing = json.load(open(timing_path)) if os.path.exists(timing_path) else {}

    ext_path = os.path.join(wdir, "ext.npy")
    if not os.path.exists(ext_path):
        t0, c0 = time.time(), time.process_time()
        ext = oracle.ext_full(x)
        timing["ext_full"] = {"wall_s": time.time() - t0, "cpu_s": time.process_time() - c0}
        np.save(ext_path + ".tmp.npy", ext)
        os.replace(ext_path + ".tmp.npy", ext_path)
        json.dump(timing, open(timing_path, "w"))
    ext = np.load(ext_path)

    nchunks = (n + chunk - 1) // chunk
    for c in range(nchunks):
        path = os.path.join(wdir, f"rows_{c:05d}.npy")
        if os.path.exists(path):
            continue
        lo, hi = c * chunk, min(n, (c + 1) * chunk)
        t0, c0 = time.time(), time.process_time()
        rows = oracle.rows_b(x, np.arange(lo, hi, dtype=np.int64))
        timing[f"chunk_{c:05d}"] = {"wall_s": time.time() - t0, "cpu_s": time.process_time() - c0,
                                    "points": hi - lo}
        np.save(path + ".tmp.npy", rows)
        os.replace(path + ".tmp.npy", path)
        json.dump(timing, open(timing_path, "w"))
        done = c + 1
        walls = [v["wall_s"] for k, v in timing.items() if k.startswith("chunk_")]
        print(f"[{name}] chunk {done}/{nchunks}  {walls[-1]:.1f}s  "
              f"(eta {np.mean(walls) * (nchunks - done) / 60:.1f} min)", flush=True)

    rows = np.empty((n, W), np.uint32)
    for c in range(nchunks):
        rows[c * chunk:min(n, (c + 1) * chunk)] = np.load(os.path.join(wdir, f"rows_{c:05d}.npy"))
    ext_ids = np.nonzero(ext)[0].astype(np.int32)
    t0 = time.time()
    offsets, ids = oracle.lattice(rows, d)
    lattice_s = time.time() - t0
    walls = [v["wall_s"] for k, v in timing.items() if k.startswith("chunk_")]
    rec = {
        "dist": cfg.dist, "n": n, "d": d, "seed": cfg.seed,
        "data": sha(x),
        "n_ext": int(ext_ids.size),
        "ext_ids": sha(ext_ids),
        "rows": sha(rows),
        "row_block": BLOCK,
        "row_blocks": [sha(rows[i:i + BLOCK]) for i in range(0, n, BLOCK)],
        "offsets": sha(offsets),
        "total_ids": int(offsets[-1]),
        "ids": sha(ids),
        "oracle": {"function": "oracle.rows_b (Oracle B) over every point; oracle.ext_full; oracle.lattice",
                   "source_sha256": file_sha(os.path.join(ROOT, "oracle", "skycube_oracle.c")),
                   "threads": threads, "cpu_model": cpu_model(),
                   "rows_b_wall_s": round(float(np.sum(walls)), 1),
                   "ext_full_wall_s": round(timing.get("ext_full", {}).get("wall_s", float("nan")), 1),
                   "lattice_wall_s": round(lattice_s, 1)},
    }
    if d <= 12:
        rec["subspace_sizes"] = np.diff(offsets).tolist()
    return rec


def main() -> None:
    ap = argparse.ArgumentParser()
    ap.add_argument("configs", nargs="+")
    ap.add_argument("--chunk", type=int, default=CHUNK)
    a = ap.parse_args()
    for name in a.configs:
        rec = run(name, a.chunk)
        g = load_golden()
        g["configs"][name] = rec
        save_golden(g)
        print(f"[{name}] n_ext={rec['n_ext']} total_ids={rec['total_ids']} rows={rec['rows'][:16]}",
              flush=True)


if __name__ == "__main__":
    main()

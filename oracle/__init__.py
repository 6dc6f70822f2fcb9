"""CPU oracle for the MDMC skycube — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and
``--impl reference``) may import this package.  The product path
(``paper_conf_sigmod_boghcsa17_b200``) never imports it and shares no code with it.

The arithmetic lives in ``skycube_oracle.c`` (Def. 1-3 of PAPER.md L92-110, written out; see the
header of that file).  This module only compiles it with gcc and marshals numpy arrays.

Functions
---------
rows_a(x)            Oracle A (literal per-subspace definition): (membership rows, extended rows)
rows_b(x, pids)      Oracle B (per point, all of P, superset closures)
cells_a(x, p, delta) Oracle A on individual (point, subspace) cells
ext_full(x)          S+(P), Alg. 3 line 2 (L320)
lattice(rows, d)     CSR lattice (Fig. 1a) from rows: offsets[2^d+1], ids ascending per subspace

Parity status: every function is pinned by tests/test_oracle_*.py (no "parity unpinned" entries).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "skycube_oracle.c")
_LIB = os.path.join(_HERE, "libskycube_oracle.so")
_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle with gcc -O2 -fopenmp (plain C, no GPU).

    ``SKYCUBE_ORACLE_CFLAGS`` (space-separated) replaces ``-O2`` and builds a separately named
    library; ``tools/oracle_digest.py`` uses ``-O3 -march=native -funroll-loops`` for its multi-hour
    full-size runs.  The source, and so the arithmetic, is the same (no -ffast-math: the oracle's only
    operations on values are IEEE ``<`` / ``<=``).  Timed baselines (bench.py) use the default."""
    flags = os.environ.get("SKYCUBE_ORACLE_CFLAGS", "").split() or ["-O2"]
    lib = _LIB if flags == ["-O2"] else _LIB.replace(
        ".so", "_" + "".join(c for c in "".join(flags) if c.isalnum()) + ".so")
    if force or not os.path.exists(lib) or os.path.getmtime(lib) < os.path.getmtime(_SRC):
        tmp = lib + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *flags, "-fopenmp", "-fPIC", "-shared", "-std=c11",
                               "-o", tmp, _SRC])
        os.replace(tmp, lib)
    return lib


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(build())
            P = ctypes.c_void_p
            I64 = ctypes.c_int64
            I32 = ctypes.c_int
            lib.oracle_a_rows.argtypes = [P, I64, I32, P, P]
            lib.oracle_a_cells.argtypes = [P, I64, I32, P, P, I64, P]
            lib.oracle_ext_full.argtypes = [P, I64, I32, P]
            lib.oracle_b_rows.argtypes = [P, I64, I32, P, I64, P, P]
            lib.oracle_lattice.argtypes = [P, I64, I32, P, P]
            for f in (lib.oracle_a_rows, lib.oracle_a_cells, lib.oracle_ext_full,
                      lib.oracle_b_rows, lib.oracle_lattice, lib.oracle_num_threads):
                f.restype = ctypes.c_int
            _lib = lib
    return _lib


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p) if a is not None else None


def _pts(x):
    x = np.ascontiguousarray(x, dtype=np.float32)
    if x.ndim != 2:
        raise ValueError("points must be (n, d)")
    if np.isnan(x).any():
        raise ValueError("NaN in points (reading Q11: NaN is an error)")
    return x


def words_per_row(d: int) -> int:
    return max(1, (1 << d) >> 5)


def num_threads() -> int:
    return _load().oracle_num_threads()


def rows_a(x, with_ext: bool = True):
    x = _pts(x)
    n, d = x.shape
    W = words_per_row(d)
    rows = np.zeros((n, W), np.uint32)
    ext = np.zeros((n, W), np.uint32) if with_ext else None
    if _load().oracle_a_rows(_ptr(x), n, d, _ptr(rows), _ptr(ext)) != 0:
        raise RuntimeError("oracle_a_rows failed")
    return (rows, ext) if with_ext else rows


def rows_b(x, pids=None, with_ext: bool = False):
    x = _pts(x)
    n, d = x.shape
    W = words_per_row(d)
    if pids is not None:
        pids = np.ascontiguousarray(pids, dtype=np.int64)
        npts = pids.shape[0]
    else:
        npts = n
    rows = np.zeros((npts, W), np.uint32)
    ext = np.zeros((npts, W), np.uint32) if with_ext else None
    if _load().oracle_b_rows(_ptr(x), n, d, _ptr(pids), npts, _ptr(rows), _ptr(ext)) != 0:
        raise RuntimeError("oracle_b_rows failed")
    return (rows, ext) if with_ext else rows


def cells_a(x, pids, deltas):
    x = _pts(x)
    n, d = x.shape
    pids = np.ascontiguousarray(pids, dtype=np.int64)
    deltas = np.ascontiguousarray(deltas, dtype=np.uint32)
    out = np.zeros(pids.shape[0], np.uint8)
    if _load().oracle_a_cells(_ptr(x), n, d, _ptr(pids), _ptr(deltas), pids.shape[0], _ptr(out)) != 0:
        raise RuntimeError("oracle_a_cells failed")
    return out.astype(bool)


def ext_full(x):
    x = _pts(x)
    n, d = x.shape
    out = np.zeros(n, np.uint8)
    if _load().oracle_ext_full(_ptr(x), n, d, _ptr(out)) != 0:
        raise RuntimeError("oracle_ext_full failed")
    return out.astype(bool)


def lattice(rows, d: int):
    rows = np.ascontiguousarray(rows, dtype=np.uint32)
    n = rows.shape[0]
    offsets = np.zeros((1 << d) + 1, np.int64)
    lib = _load()
    if lib.oracle_lattice(_ptr(rows), n, d, _ptr(offsets), None) != 0:
        raise RuntimeError("oracle_lattice failed")
    ids = np.zeros(int(offsets[-1]), np.int32)
    if lib.oracle_lattice(_ptr(rows), n, d, _ptr(offsets), _ptr(ids)) != 0:
        raise RuntimeError("oracle_lattice failed")
    return offsets, ids


def row_bit(rows, p: int, delta: int) -> bool:
    return bool((int(rows[p, delta >> 5]) >> (delta & 31)) & 1)


def skycube(x, method: str = "b"):
    """Full oracle skycube: dict(rows, ext_ids, offsets, ids) with the C-ABI's conventions."""
    x = _pts(x)
    n, d = x.shape
    rows = rows_a(x, with_ext=False) if method == "a" else rows_b(x)
    ext = ext_full(x)
    offsets, ids = lattice(rows, d)
    return {"rows": rows, "ext_ids": np.nonzero(ext)[0].astype(np.int32),
            "offsets": offsets, "ids": ids}

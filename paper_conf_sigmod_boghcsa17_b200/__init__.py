"""B200-native point-based MDMC skycube (Bøgh et al., SIGMOD'17) — thin Python binding.

The binding only marshals arguments to the C-ABI of ``include/skycube.h`` (``libskycube.so``, built
in-tree by ``paper_conf_sigmod_boghcsa17_b200.build``).  Every step of the skycube runs in the CUDA
kernels of ``csrc/``; there is no CPU fallback: if the library or an sm_100 GPU is missing, calls
raise.  PyTorch is only used by callers for device memory, streams and process groups.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SKYCUBE_LIB") or os.path.join(_PKG, "libskycube.so")

OK, EINVAL, ENAN, ENOMEM, ECUDA, ENCCL, ENODEV = range(7)
NO_LISTS = 0x1
EXT_MEMBERSHIP = 0x2

EXPORTED = (
    "skycube_build", "skycube_build_ex", "skycube_free", "skycube_strerror", "skycube_last_error",
    "skycube_ctx_create", "skycube_ctx_destroy", "skycube_dev_prepare", "skycube_dev_prefilter",
    "skycube_dev_set_ext", "skycube_dev_mdmc", "skycube_dev_compact", "skycube_ctx_launches",
    "skycube_ctx_info", "skycube_ctx_counters", "skycube_build_hashcube", "skycube_hashcube_free",
    "skycube_hashcube_query", "skycube_ctx_set_max_level", "skycube_dev_hashcube", "skycube_build_sdsc",
    "skycube_set_tuning", "skycube_dev_lattice_count", "skycube_dev_lattice_scatter", "skycube_dev_membership",
    "skycube_dev_prepare_dims", "skycube_dev_prepare_finish",
)


class SkycubeError(RuntimeError):
    def __init__(self, status, detail):
        super().__init__(f"skycube status {status}: {detail}")
        self.status = status


class Result(ctypes.Structure):
    _fields_ = [
        ("d", ctypes.c_int32),
        ("n", ctypes.c_int64),
        ("n_ext", ctypes.c_int64),
        ("ext_ids", ctypes.POINTER(ctypes.c_int32)),
        ("words_per_row", ctypes.c_uint32),
        ("membership", ctypes.POINTER(ctypes.c_uint32)),
        ("ext_membership", ctypes.POINTER(ctypes.c_uint32)),
        ("cuboid_offsets", ctypes.POINTER(ctypes.c_int64)),
        ("cuboid_ids", ctypes.POINTER(ctypes.c_int32)),
    ]


class Opts(ctypes.Structure):
    _fields_ = [("num_gpus", ctypes.c_int32), ("device", ctypes.c_int32), ("flags", ctypes.c_uint32),
                ("max_level", ctypes.c_int32)]


class HashCube(ctypes.Structure):
    _fields_ = [
        ("d", ctypes.c_int32), ("w", ctypes.c_uint32), ("n", ctypes.c_int64), ("n_ext", ctypes.c_int64),
        ("n_words", ctypes.c_int64), ("total_keys", ctypes.c_int64), ("total_ids", ctypes.c_int64),
        ("word_offsets", ctypes.POINTER(ctypes.c_int64)), ("keys", ctypes.POINTER(ctypes.c_uint32)),
        ("key_offsets", ctypes.POINTER(ctypes.c_int64)), ("ids", ctypes.POINTER(ctypes.c_int32)),
    ]


class Stats(ctypes.Structure):
    _fields_ = [(k, ctypes.c_double) for k in ("ms_total", "ms_h2d", "ms_validate", "ms_sort", "ms_codes",
                                                "ms_prefilter", "ms_mdmc", "ms_compact", "ms_d2h")] + [
        ("n_ext", ctypes.c_int64), ("pairs", ctypes.c_int64), ("total_ids", ctypes.c_int64),
        ("kernel_launches", ctypes.c_int32), ("ms_comm", ctypes.c_double), ("exact_dts", ctypes.c_int64),
        ("expansions", ctypes.c_int64), ("num_gpus", ctypes.c_int32)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


_lib = None


def lib():
    """Load libskycube.so; raises (never falls back) if it is missing."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} not built: run python -m paper_conf_sigmod_boghcsa17_b200.build")
        L = ctypes.CDLL(LIB_PATH)
        P, I64, I32, U32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_uint32
        L.skycube_build.argtypes = [P, I64, I32, ctypes.POINTER(Result)]
        L.skycube_build_ex.argtypes = [P, I64, I32, ctypes.POINTER(Opts), ctypes.POINTER(Result),
                                       ctypes.POINTER(Stats)]
        L.skycube_free.argtypes = [ctypes.POINTER(Result)]
        L.skycube_free.restype = None
        L.skycube_strerror.argtypes = [ctypes.c_int]
        L.skycube_strerror.restype = ctypes.c_char_p
        L.skycube_last_error.restype = ctypes.c_char_p
        L.skycube_ctx_create.argtypes = [I32, ctypes.POINTER(P)]
        L.skycube_ctx_destroy.argtypes = [P]
        L.skycube_ctx_destroy.restype = None
        L.skycube_dev_prepare.argtypes = [P, P, I64, I32, P]
        L.skycube_dev_prepare_dims.argtypes = [P, P, I64, I32, I32, I32, P, P, P, P]
        L.skycube_dev_prepare_finish.argtypes = [P, P, P, P, P]
        L.skycube_dev_prefilter.argtypes = [P, I64, I64, P, P]
        L.skycube_dev_set_ext.argtypes = [P, P, ctypes.POINTER(I64), P]
        L.skycube_dev_mdmc.argtypes = [P, I64, I64, P, P, P]
        L.skycube_dev_compact.argtypes = [P, P, P, P, P, P, ctypes.POINTER(I64), P]
        L.skycube_ctx_launches.argtypes = [P]
        L.skycube_ctx_launches.restype = I64
        L.skycube_ctx_info.argtypes = [P, ctypes.POINTER(I64), ctypes.POINTER(U32), ctypes.POINTER(U32)]
        L.skycube_ctx_counters.argtypes = [P, P]
        L.skycube_build_sdsc.argtypes = [P, I64, I32, ctypes.POINTER(Opts), ctypes.POINTER(Result),
                                          ctypes.POINTER(Stats)]
        L.skycube_build_hashcube.argtypes = [P, I64, I32, U32, ctypes.POINTER(Opts), ctypes.POINTER(HashCube),
                                             ctypes.POINTER(Stats)]
        L.skycube_hashcube_free.argtypes = [ctypes.POINTER(HashCube)]
        L.skycube_hashcube_free.restype = None
        L.skycube_hashcube_query.argtypes = [ctypes.POINTER(HashCube), U32, P, ctypes.POINTER(I64)]
        L.skycube_ctx_set_max_level.argtypes = [P, I32]
        L.skycube_dev_hashcube.argtypes = [P, P, U32, P, P, P, P, ctypes.POINTER(I64), ctypes.POINTER(I64),
                                           ctypes.POINTER(I64), P]
        L.skycube_set_tuning.argtypes = [ctypes.c_char_p, I32]
        L.skycube_dev_lattice_count.argtypes = [P, P, I64, I64, P, P]
        L.skycube_dev_lattice_scatter.argtypes = [P, P, I64, I64, P, I32, I32, P, P, ctypes.POINTER(I64), P]
        L.skycube_dev_membership.argtypes = [P, P, I64, I64, I64, I64, P, P]
        for f in ("skycube_dev_lattice_count", "skycube_dev_lattice_scatter", "skycube_dev_membership",
                  "skycube_dev_prepare_dims", "skycube_dev_prepare_finish",
                  "skycube_set_tuning", "skycube_build", "skycube_build_ex", "skycube_ctx_create", "skycube_dev_prepare",
                  "skycube_dev_prefilter", "skycube_dev_set_ext", "skycube_dev_mdmc", "skycube_dev_compact",
                  "skycube_ctx_info", "skycube_ctx_counters", "skycube_build_hashcube", "skycube_hashcube_query",
                  "skycube_ctx_set_max_level", "skycube_dev_hashcube", "skycube_build_sdsc"):
            getattr(L, f).restype = ctypes.c_int
        _lib = L
        # tools/*.sh A/B runs name tuning overrides in the environment; applied once, here, never in the
        # library's launch path
        for key, env in (("k3_design", "SKYCUBE_K3_DESIGN"), ("k3_tpc", "SKYCUBE_K3_TPC"), ("k3_warps", "SKYCUBE_K3_WARPS"),
                         ("k3_mode", "SKYCUBE_K3_MODE"), ("share_devices", "SKYCUBE_SHARE_DEVICES")):
            v = os.environ.get(env, "")
            if v:
                set_tuning(key, ord(v[0]) if key == "k3_design" else int(v))
    return _lib


def set_tuning(key: str, value: int) -> None:
    """skycube_set_tuning: performance-only overrides (k3_design 'A'/'O' as ord(), k3_tpc, k3_mode,
    share_devices) or key "reset"."""
    if isinstance(value, str):
        value = ord(value[0])
    _check(lib().skycube_set_tuning(key.encode(), int(value)))


def _check(status):
    if status != OK:
        raise SkycubeError(status, lib().skycube_last_error().decode(errors="replace"))


def words_per_row(d: int) -> int:
    return max(1, (1 << d) >> 5)


def _view(ptr, count, dtype):
    if count <= 0 or not ptr:
        return np.zeros(0, dtype)
    return np.ctypeslib.as_array(ptr, shape=(count,)).view(dtype)


class RawResult:
    """Owns a skycube_result (pinned host buffers); views are valid until close()."""

    def __init__(self, res: Result, stats: Stats | None):
        self._res = res
        self.stats = stats.as_dict() if stats is not None else None

    @property
    def n(self):
        return self._res.n

    @property
    def d(self):
        return self._res.d

    @property
    def n_ext(self):
        return self._res.n_ext

    def ext_ids(self):
        return _view(self._res.ext_ids, self._res.n_ext, np.int32)

    def membership(self):
        W = self._res.words_per_row
        return _view(self._res.membership, self._res.n * W, np.uint32).reshape(self._res.n, W)

    def ext_membership(self):
        W = self._res.words_per_row
        if not self._res.ext_membership:
            return None
        return _view(self._res.ext_membership, self._res.n * W, np.uint32).reshape(self._res.n, W)

    def offsets(self):
        if not self._res.cuboid_offsets:
            return None
        return _view(self._res.cuboid_offsets, (1 << self._res.d) + 1, np.int64)

    def ids(self):
        off = self.offsets()
        if off is None:
            return None
        return _view(self._res.cuboid_ids, int(off[-1]), np.int32)

    def close(self):
        if self._res is not None:
            lib().skycube_free(ctypes.byref(self._res))
            self._res = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def skycube_build_raw(points: np.ndarray, *, device: int = 0, lists: bool = True, ext_membership: bool = False,
                      stats: bool = False, max_level: int = 0, num_gpus: int = 1) -> RawResult:
    """Call skycube_build_ex on a host (n, d) float32 array; returns the owning RawResult.
    max_level = d' > 0 computes the partial skycube (|delta| <= d' only, Appendix A.2)."""
    pts = np.ascontiguousarray(points, dtype=np.float32)
    if pts.ndim != 2:
        raise ValueError("points must be (n, d)")
    n, d = pts.shape
    opts = Opts(num_gpus, device, (0 if lists else NO_LISTS) | (EXT_MEMBERSHIP if ext_membership else 0), max_level)
    res = Result()
    st = Stats() if stats else None
    _check(lib().skycube_build_ex(pts.ctypes.data_as(ctypes.c_void_p) if n else None, n, d, ctypes.byref(opts),
                                  ctypes.byref(res), ctypes.byref(st) if st is not None else None))
    return RawResult(res, st)


def skycube_build(points: np.ndarray, **kw) -> dict:
    """Skycube of a host (n, d) float32 array, copied into numpy arrays:
    rows [n, W] uint32 (bit delta <=> point in S_delta), ext_ids, offsets [2^d+1], ids."""
    with skycube_build_raw(points, **kw) as r:
        out = {"rows": r.membership().copy(), "ext_ids": r.ext_ids().copy(), "n_ext": r.n_ext}
        off = r.offsets()
        if off is not None:
            out["offsets"] = off.copy()
            out["ids"] = r.ids().copy()
        em = r.ext_membership()
        if em is not None:
            out["ext_rows"] = em.copy()
        if r.stats is not None:
            out["stats"] = r.stats
        return out


def skycube_build_sdsc(points: np.ndarray, *, device: int = 0, stats: bool = False) -> dict:
    """The SDSC comparator (Alg. 2) through skycube_build_sdsc: same dict as skycube_build."""
    pts = np.ascontiguousarray(points, dtype=np.float32)
    if pts.ndim != 2:
        raise ValueError("points must be (n, d)")
    n, d = pts.shape
    opts = Opts(1, device, 0, 0)
    res = Result()
    st = Stats() if stats else None
    _check(lib().skycube_build_sdsc(pts.ctypes.data_as(ctypes.c_void_p) if n else None, n, d, ctypes.byref(opts),
                                    ctypes.byref(res), ctypes.byref(st) if st is not None else None))
    with RawResult(res, st) as r:
        out = {"rows": r.membership().copy(), "ext_ids": r.ext_ids().copy(), "n_ext": r.n_ext,
               "offsets": r.offsets().copy(), "ids": r.ids().copy()}
        if r.stats is not None:
            out["stats"] = r.stats
        return out


class RawHashCube:
    """Owns a skycube_hashcube (pinned host buffers); views are valid until close()."""

    def __init__(self, hc: HashCube, stats: Stats | None):
        self._hc = hc
        self.stats = stats.as_dict() if stats is not None else None

    def arrays(self) -> dict:
        h = self._hc
        return {"word_offsets": _view(h.word_offsets, h.n_words + 1, np.int64),
                "keys": _view(h.keys, h.total_keys, np.uint32),
                "key_offsets": _view(h.key_offsets, h.total_keys + 1, np.int64),
                "ids": _view(h.ids, h.total_ids, np.int32)}

    def query(self, delta: int) -> np.ndarray:
        """S_delta(P) ascending, through skycube_hashcube_query (L1280)."""
        cnt = ctypes.c_int64()
        _check(lib().skycube_hashcube_query(ctypes.byref(self._hc), delta, None, ctypes.byref(cnt)))
        out = np.zeros(max(cnt.value, 1), np.int32)
        _check(lib().skycube_hashcube_query(ctypes.byref(self._hc), delta, out.ctypes.data_as(ctypes.c_void_p),
                                            ctypes.byref(cnt)))
        return out[:cnt.value]

    @property
    def n_ext(self):
        return self._hc.n_ext

    def close(self):
        if self._hc is not None:
            lib().skycube_hashcube_free(ctypes.byref(self._hc))
            self._hc = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def skycube_build_hashcube_raw(points: np.ndarray, w: int = 32, *, device: int = 0, max_level: int = 0,
                               stats: bool = False) -> RawHashCube:
    """Call skycube_build_hashcube (HashCube output, Appendix B.1) on a host (n, d) float32 array."""
    pts = np.ascontiguousarray(points, dtype=np.float32)
    if pts.ndim != 2:
        raise ValueError("points must be (n, d)")
    n, d = pts.shape
    opts = Opts(1, device, 0, max_level)
    hc = HashCube()
    st = Stats() if stats else None
    _check(lib().skycube_build_hashcube(pts.ctypes.data_as(ctypes.c_void_p) if n else None, n, d, w,
                                        ctypes.byref(opts), ctypes.byref(hc),
                                        ctypes.byref(st) if st is not None else None))
    return RawHashCube(hc, st)


def skycube_build_hashcube(points: np.ndarray, w: int = 32, **kw) -> dict:
    """HashCube of a host (n, d) float32 array, copied into numpy arrays (word_offsets, keys, key_offsets,
    ids) plus n_ext."""
    with skycube_build_hashcube_raw(points, w, **kw) as r:
        out = {k: v.copy() for k, v in r.arrays().items()}
        out["n_ext"] = r.n_ext
        if r.stats is not None:
            out["stats"] = r.stats
        return out


@dataclass
class Context:
    """Device-level API (device pointers as ints, e.g. torch tensor .data_ptr(); stream as int)."""

    device: int = 0

    def __post_init__(self):
        h = ctypes.c_void_p()
        _check(lib().skycube_ctx_create(self.device, ctypes.byref(h)))
        self._h = h

    def close(self):
        if getattr(self, "_h", None):
            lib().skycube_ctx_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def prepare(self, d_points: int, n: int, d: int, stream: int = 0):
        _check(lib().skycube_dev_prepare(self._h, d_points, n, d, stream or None))

    def prepare_dims(self, d_points: int, n: int, d: int, dim_begin: int, dim_end: int, d_codes_dm: int, d_R: int,
                     d_minord: int, stream: int = 0):
        _check(lib().skycube_dev_prepare_dims(self._h, d_points, n, d, dim_begin, dim_end, d_codes_dm or None,
                                              d_R or None, d_minord or None, stream or None))

    def prepare_finish(self, d_codes_dm: int, d_R: int, d_minord: int, stream: int = 0):
        _check(lib().skycube_dev_prepare_finish(self._h, d_codes_dm, d_R, d_minord, stream or None))

    def prefilter(self, d_ext_sorted: int, tile_offset: int = 0, tile_step: int = 1, stream: int = 0):
        _check(lib().skycube_dev_prefilter(self._h, tile_offset, tile_step, d_ext_sorted, stream or None))

    def set_ext(self, d_ext_sorted: int, stream: int = 0) -> int:
        m = ctypes.c_int64()
        _check(lib().skycube_dev_set_ext(self._h, d_ext_sorted, ctypes.byref(m), stream or None))
        return m.value

    def mdmc(self, d_rows32: int, j_begin: int, j_end: int, d_ext_rows32: int = 0, stream: int = 0):
        _check(lib().skycube_dev_mdmc(self._h, j_begin, j_end, d_rows32, d_ext_rows32 or None, stream or None))

    def compact(self, d_rows32: int, d_membership: int = 0, d_ext_ids: int = 0, d_offsets: int = 0,
                d_ids: int = 0, stream: int = 0) -> int:
        tot = ctypes.c_int64(0)
        _check(lib().skycube_dev_compact(self._h, d_rows32, d_membership or None, d_ext_ids or None,
                                         d_offsets or None, d_ids or None, ctypes.byref(tot), stream or None))
        return tot.value

    def lattice_count(self, d_rows32: int, j_begin: int, j_end: int, d_totals: int, stream: int = 0):
        """Per-subspace counts of the S+ tasks [j_begin, j_end) -> d_totals[2^d] (int64 device)."""
        _check(lib().skycube_dev_lattice_count(self._h, d_rows32, j_begin, j_end, d_totals, stream or None))

    def lattice_scatter(self, d_rows32: int, j_begin: int, j_end: int, d_all_totals: int, num_shards: int, shard: int,
                        d_offsets: int = 0, ids: int = 0, stream: int = 0) -> int:
        """Global offsets and this shard's ids at their global positions (ids: device or host-mapped pointer);
        returns the global id count."""
        tot = ctypes.c_int64(0)
        _check(lib().skycube_dev_lattice_scatter(self._h, d_rows32, j_begin, j_end, d_all_totals, num_shards, shard,
                                                 d_offsets or None, ids or None, ctypes.byref(tot), stream or None))
        return tot.value

    def membership(self, d_rows32: int, j_begin: int, j_end: int, zero_lo: int, zero_hi: int, membership: int,
                   stream: int = 0):
        """Rows of the S+ tasks [j_begin, j_end) by id + zero rows outside S+ for ids in [zero_lo, zero_hi)."""
        _check(lib().skycube_dev_membership(self._h, d_rows32, j_begin, j_end, zero_lo, zero_hi, membership,
                                            stream or None))

    def set_max_level(self, max_level: int):
        _check(lib().skycube_ctx_set_max_level(self._h, max_level))

    def hashcube(self, d_rows32: int, w: int, stream: int = 0):
        """Build the HashCube in the context workspace: returns (n_words, total_keys, total_ids)."""
        nw, nk, ni = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
        _check(lib().skycube_dev_hashcube(self._h, d_rows32, w, None, None, None, None, ctypes.byref(nw),
                                          ctypes.byref(nk), ctypes.byref(ni), stream or None))
        return nw.value, nk.value, ni.value

    def hashcube_copy(self, w: int, d_word_offsets: int, d_keys: int, d_key_offsets: int, d_ids: int,
                      stream: int = 0):
        _check(lib().skycube_dev_hashcube(self._h, None, w, d_word_offsets, d_keys, d_key_offsets, d_ids,
                                          None, None, None, stream or None))

    @property
    def launches(self) -> int:
        return lib().skycube_ctx_launches(self._h)

    def counters(self) -> dict:
        a = np.zeros(8, np.int64)
        _check(lib().skycube_ctx_counters(self._h, a.ctypes.data_as(ctypes.c_void_p)))
        return {"k1_box": int(a[0]), "k1_pair": int(a[1]), "k3_box": int(a[2]), "k3_pair": int(a[3]),
                "k3_miss": int(a[4]), "k3_sub": int(a[5]), "k3_expansions": int(a[6])}

    def info(self):
        m, W, ex = ctypes.c_int64(), ctypes.c_uint32(), ctypes.c_uint32()
        _check(lib().skycube_ctx_info(self._h, ctypes.byref(m), ctypes.byref(W), ctypes.byref(ex)))
        return {"n_ext": m.value, "words_per_row": W.value, "exact_mask": ex.value}

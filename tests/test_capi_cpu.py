"""CPU-side checks of the C-ABI library: it builds, loads, exports every declared symbol, and validates
arguments without touching a GPU (no compute calls here)."""
from __future__ import annotations

import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_sigmod_boghcsa17_b200 as sky
from paper_conf_sigmod_boghcsa17_b200 import build as skybuild

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared_functions():
    text = open(os.path.join(ROOT, "include", "skycube.h")).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(skycube_\w+)\s*\(", text)))


@pytest.fixture(scope="module")
def lib():
    skybuild.build()
    return sky.lib()


def test_header_declares_expected_api():
    decl = _declared_functions()
    assert set(sky.EXPORTED) == set(decl), (sorted(set(decl) ^ set(sky.EXPORTED)))


def test_library_exports_every_declared_symbol(lib):
    for name in _declared_functions():
        assert hasattr(lib, name), name
    # and they are real dynamic symbols of libskycube.so
    out = os.popen(f"nm -D --defined-only {sky.LIB_PATH}").read()
    for name in _declared_functions():
        assert re.search(rf"\bT {name}$", out, flags=re.M), name


def test_sm100a_cubin_only(lib):
    out = os.popen(f"/usr/local/cuda/bin/cuobjdump --list-elf {sky.LIB_PATH}").read()
    assert "sm_100a" in out
    assert not re.search(r"sm_(?!100a)\d+", out), out


def test_strerror(lib):
    assert lib.skycube_strerror(0) == b"ok"
    assert lib.skycube_strerror(sky.ENAN) == b"NaN in input"


def test_argument_validation_without_gpu(lib):
    res = sky.Result()
    pts = np.zeros((4, 3), np.float32)
    p = pts.ctypes.data_as(ctypes.c_void_p)
    assert lib.skycube_build(p, 4, 0, ctypes.byref(res)) == sky.EINVAL
    assert lib.skycube_build(p, 4, 17, ctypes.byref(res)) == sky.EINVAL
    assert lib.skycube_build(None, 4, 3, ctypes.byref(res)) == sky.EINVAL
    assert lib.skycube_build(p, -1, 3, ctypes.byref(res)) == sky.EINVAL
    assert lib.skycube_build(p, 1 << 31, 3, ctypes.byref(res)) == sky.EINVAL
    assert lib.skycube_build(p, 4, 3, None) == sky.EINVAL
    assert res.membership is None or not res.membership
    lib.skycube_free(ctypes.byref(res))
    lib.skycube_free(None)


def test_no_cpu_fallback_without_gpu(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    res = sky.Result()
    pts = np.zeros((4, 3), np.float32)
    st = lib.skycube_build(pts.ctypes.data_as(ctypes.c_void_p), 4, 3, ctypes.byref(res))
    assert st == sky.ENODEV
    assert b"device" in lib.skycube_last_error()


def test_hashcube_and_partial_validation_without_gpu(lib):
    pts = np.zeros((4, 3), np.float32)
    p = pts.ctypes.data_as(ctypes.c_void_p)
    hc = sky.HashCube()
    assert lib.skycube_build_hashcube(p, 4, 3, 0, None, ctypes.byref(hc), None) == sky.EINVAL
    assert lib.skycube_build_hashcube(p, 4, 3, 33, None, ctypes.byref(hc), None) == sky.EINVAL
    assert lib.skycube_build_hashcube(p, 4, 17, 32, None, ctypes.byref(hc), None) == sky.EINVAL
    opts = sky.Opts(1, 0, 0, 4)  # max_level > d
    res = sky.Result()
    assert lib.skycube_build_ex(p, 4, 3, ctypes.byref(opts), ctypes.byref(res), None) == sky.EINVAL
    cnt = ctypes.c_int64()
    assert lib.skycube_hashcube_query(ctypes.byref(sky.HashCube()), 1, None, ctypes.byref(cnt)) == sky.EINVAL
    lib.skycube_hashcube_free(ctypes.byref(hc))  # safe on a zeroed struct


def test_hashcube_query_host_logic_fig1b(lib):
    """The read path (skycube_hashcube_query, host code) on the Fig. 1b HashCube built by the oracle."""
    import json
    import oracle
    from oracle import hashcube as hco
    gold = json.load(open(os.path.join(ROOT, "tests", "golden", "flights.json")))
    x = np.array(gold["points"], np.float32)
    for w in (4, 1, 3, 32):
        a = hco.hashcube(oracle.rows_a(x, with_ext=False), 3, w)
        hc = sky.HashCube()
        hc.d, hc.w, hc.n, hc.n_words = 3, w, 5, hco.n_words(3, w)
        hc.total_keys, hc.total_ids = a["keys"].size, a["ids"].size
        hc.word_offsets = a["word_offsets"].ctypes.data_as(ctypes.POINTER(ctypes.c_int64))
        hc.keys = a["keys"].ctypes.data_as(ctypes.POINTER(ctypes.c_uint32))
        hc.key_offsets = a["key_offsets"].ctypes.data_as(ctypes.POINTER(ctypes.c_int64))
        hc.ids = a["ids"].ctypes.data_as(ctypes.POINTER(ctypes.c_int32))
        for delta in range(1, 8):
            cnt = ctypes.c_int64()
            assert lib.skycube_hashcube_query(ctypes.byref(hc), delta, None, ctypes.byref(cnt)) == sky.OK
            out = np.zeros(max(1, cnt.value), np.int32)
            assert lib.skycube_hashcube_query(ctypes.byref(hc), delta, out.ctypes.data_as(ctypes.c_void_p),
                                              ctypes.byref(cnt)) == sky.OK
            assert out[:cnt.value].tolist() == gold["lattice"][str(delta)], (w, delta)
        assert lib.skycube_hashcube_query(ctypes.byref(hc), 8, None, ctypes.byref(cnt)) == sky.EINVAL


def test_num_gpus_validation_without_gpu(lib):
    pts = np.zeros((4, 3), np.float32)
    p = pts.ctypes.data_as(ctypes.c_void_p)
    res = sky.Result()
    assert lib.skycube_build_ex(p, 4, 3, ctypes.byref(sky.Opts(-1, 0, 0, 0)), ctypes.byref(res), None) == sky.EINVAL
    assert lib.skycube_build_ex(p, 4, 3, ctypes.byref(sky.Opts(2, 0, sky.EXT_MEMBERSHIP, 0)), ctypes.byref(res),
                                None) == sky.EINVAL
    # no device in this container: the multi-GPU path reports ENODEV, never a CPU fallback
    assert lib.skycube_build_ex(p, 4, 3, ctypes.byref(sky.Opts(2, 0, 0, 0)), ctypes.byref(res), None) == sky.ENODEV

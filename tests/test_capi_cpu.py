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

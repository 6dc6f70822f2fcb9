"""The SDSC comparator (Alg. 2 on the GPU, skycube_build_sdsc) against the CPU oracles: bit-exact lattice,
membership rows and S+ ids (Oracle B / Oracle A), plus agreement with the MDMC product path.  Needs a B200."""
from __future__ import annotations

import json
import os

import numpy as np
import pytest

import datagen
import oracle
from oracle import sdsc as osdsc
import paper_conf_sigmod_boghcsa17_b200 as sky

pytestmark = pytest.mark.gpu

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "flights.json")))


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    sky.lib()


def check(x):
    n, d = x.shape
    r = sky.skycube_build_sdsc(x)
    want = oracle.rows_b(x)
    bad = np.nonzero((r["rows"] != want).any(axis=1))[0]
    assert bad.size == 0, f"{bad.size} rows differ, first {bad[:5]}"
    off, ids = oracle.lattice(want, d)
    assert np.array_equal(r["offsets"], off) and np.array_equal(r["ids"], ids)
    assert np.array_equal(r["ext_ids"], np.nonzero(oracle.ext_full(x))[0])
    return r


def test_flights():
    x = np.array(GOLD["points"], np.float32)
    r = check(x)
    assert r["offsets"].tolist() == [0, 0, 1, 2, 5, 6, 9, 12, 16]


def test_alg2_literal_small():
    """The GPU traversal equals the literal Alg. 2 oracle (same parent rule) on tie-heavy data."""
    x = datagen.small_int_grid(60, 4, 3, 5)
    r = sky.skycube_build_sdsc(x)
    L, _ = osdsc.sdsc(x)
    off, ids = osdsc.to_lattice(L, 4)
    assert np.array_equal(r["offsets"], off) and np.array_equal(r["ids"], ids)


@pytest.mark.parametrize("d", [1, 2, 3, 5, 7, 9, 11])
def test_tie_heavy(d):
    check(datagen.small_int_grid(300, d, 3, 700 + d))


@pytest.mark.parametrize("case", [("A", 3000, 6, 81), ("I", 4000, 8, 82), ("C", 5000, 10, 83), ("ct", 3000, 10, 84)])
def test_continuous_and_ct(case):
    dist, n, d, seed = case
    check(datagen.generate(dist, n, d, seed))


def test_edge_cases():
    check(np.array([[1.0, 2.0]], np.float32))
    check(np.zeros((7, 3), np.float32))
    check(np.array([[0.0, 1.0], [-0.0, 1.0], [np.inf, -np.inf]], np.float32))
    r = sky.skycube_build_sdsc(np.zeros((0, 3), np.float32))
    assert r["offsets"].tolist() == [0] * 9


@pytest.mark.parametrize("name", ["C1", "C2", "C3C"])
def test_equals_mdmc_on_configs(name):
    x = datagen.config(name).data()
    a = sky.skycube_build_sdsc(x)
    b = sky.skycube_build(x)
    assert np.array_equal(a["rows"], b["rows"])
    assert np.array_equal(a["offsets"], b["offsets"]) and np.array_equal(a["ids"], b["ids"])

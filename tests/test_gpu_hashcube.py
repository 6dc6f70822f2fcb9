"""HashCube output (K5, Appendix B.1) and partial skycube (Appendix A.2) of the CUDA path against the CPU
oracle (oracle/hashcube.py over oracle rows) — bit-exact, needs a B200."""
from __future__ import annotations

import json
import os

import numpy as np
import pytest

import datagen
import oracle
from oracle import hashcube as hco
import paper_conf_sigmod_boghcsa17_b200 as sky

pytestmark = pytest.mark.gpu

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "flights.json")))
HC_GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "hashcube_fig1b.json")))


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    sky.lib()


def assert_same_hashcube(got, want):
    for k in ("word_offsets", "keys", "key_offsets", "ids"):
        assert got[k].shape == want[k].shape, (k, got[k].shape, want[k].shape)
        bad = np.nonzero(got[k] != want[k])[0]
        assert bad.size == 0, f"{k}: {bad.size} entries differ, first at {bad[:5]}"


def test_flights_fig1b():
    x = np.array(GOLD["points"], np.float32)
    hc = sky.skycube_build_hashcube(x, 4)
    assert hc["word_offsets"].tolist() == [0, 4, 7]
    h0 = {str(int(hc["keys"][u])): hc["ids"][hc["key_offsets"][u]:hc["key_offsets"][u + 1]].tolist()
          for u in range(0, 4)}
    h1 = {str(int(hc["keys"][u])): hc["ids"][hc["key_offsets"][u]:hc["key_offsets"][u + 1]].tolist()
          for u in range(4, 7)}
    assert h0 == HC_GOLD["h0"] and h1 == HC_GOLD["h1"]
    with sky.skycube_build_hashcube_raw(x, 4) as r:
        for delta in range(1, 8):
            assert r.query(delta).tolist() == GOLD["lattice"][str(delta)]


CASES = [
    ("A", 3000, 6, 31), ("A", 2500, 9, 32), ("I", 4000, 12, 33), ("A", 1500, 13, 34), ("C", 3000, 5, 35),
]


@pytest.mark.parametrize("w", [32, 4, 1, 7, 16])
@pytest.mark.parametrize("case", CASES[:3])
def test_hashcube_vs_oracle(case, w):
    dist, n, d, seed = case
    x = datagen.generate(dist, n, d, seed)
    want = hco.hashcube(oracle.rows_b(x), d, w)
    assert_same_hashcube(sky.skycube_build_hashcube(x, w), want)


@pytest.mark.parametrize("d", [1, 2, 3, 4, 5, 8, 11, 14, 16])
def test_hashcube_tie_heavy_every_shape(d):
    x = datagen.small_int_grid(120 if d < 14 else 70, d, 3, 500 + d)
    rows = oracle.rows_b(x)
    for w in (32, 5):
        assert_same_hashcube(sky.skycube_build_hashcube(x, w), hco.hashcube(rows, d, w))


def test_hashcube_query_matches_lattice():
    x = datagen.generate("A", 2000, 8, 41)
    full = sky.skycube_build(x)
    with sky.skycube_build_hashcube_raw(x, 32) as r:
        for delta in range(1, 1 << 8):
            want = full["ids"][full["offsets"][delta]:full["offsets"][delta + 1]]
            assert np.array_equal(r.query(delta), want), delta


def test_hashcube_edge_cases():
    one = np.array([[1.0, 2.0, 3.0]], np.float32)
    hc = sky.skycube_build_hashcube(one, 32)
    # a single point is in every skyline: one key 0 in the only word
    assert hc["word_offsets"].tolist() == [0, 1] and hc["keys"].tolist() == [0] and hc["ids"].tolist() == [0]
    same = np.zeros((5, 4), np.float32)
    hc = sky.skycube_build_hashcube(same, 8)
    assert_same_hashcube(hc, hco.hashcube(oracle.rows_b(same), 4, 8))
    empty = sky.skycube_build_hashcube(np.zeros((0, 3), np.float32), 4)
    assert empty["word_offsets"].tolist() == [0, 0, 0] and empty["ids"].size == 0
    with pytest.raises(sky.SkycubeError):
        sky.skycube_build_hashcube(one, 0)
    with pytest.raises(sky.SkycubeError):
        sky.skycube_build_hashcube(one, 33)


# ------------------------------------------------------------------------------- partial skycube
@pytest.mark.parametrize("case", [("A", 3000, 6, 51), ("I", 3000, 10, 52), ("A", 1200, 14, 53)])
def test_partial_vs_oracle(case):
    dist, n, d, seed = case
    x = datagen.generate(dist, n, d, seed)
    rows = oracle.rows_b(x)
    for dp in sorted({1, 2, d // 2, d - 1, d}):
        r = sky.skycube_build(x, max_level=dp)
        want = hco.partial_rows(rows, d, dp)
        bad = np.nonzero((r["rows"] != want).any(axis=1))[0]
        assert bad.size == 0, (dp, bad[:5])
        off, ids = oracle.lattice(want, d)
        assert np.array_equal(r["offsets"], off) and np.array_equal(r["ids"], ids), dp


def test_partial_tie_heavy_and_hashcube():
    x = datagen.small_int_grid(200, 9, 3, 61)
    rows = oracle.rows_b(x)
    for dp in (2, 5):
        want = hco.partial_rows(rows, 9, dp)
        assert np.array_equal(sky.skycube_build(x, max_level=dp)["rows"], want)
        assert_same_hashcube(sky.skycube_build_hashcube(x, 32, max_level=dp), hco.hashcube(want, 9, 32))


def test_partial_bad_level():
    with pytest.raises(sky.SkycubeError):
        sky.skycube_build(np.zeros((3, 3), np.float32), max_level=4)


def test_device_pipeline_hashcube_and_partial():
    """The bench launch path (pipeline.DeviceSkycube over the device entry points) gives the same bytes."""
    import torch
    from paper_conf_sigmod_boghcsa17_b200.pipeline import DeviceSkycube
    x = datagen.generate("A", 5000, 10, 71)
    rows = oracle.rows_b(x)
    eng = DeviceSkycube(0)
    out = eng.build(torch.from_numpy(x).cuda(), hashcube_w=32, max_level=6)
    want = hco.partial_rows(rows, 10, 6)
    assert np.array_equal(out["membership"].cpu().numpy().view(np.uint32), want)
    got = {k: v.cpu().numpy() for k, v in out["hashcube"].items()}
    got["keys"] = got["keys"].view(np.uint32)
    assert_same_hashcube(got, hco.hashcube(want, 10, 32))
    out = eng.build(torch.from_numpy(x).cuda())  # max_level resets to the full skycube
    assert np.array_equal(out["membership"].cpu().numpy().view(np.uint32), rows)

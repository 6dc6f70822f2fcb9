"""Pins for the HashCube and partial-skycube oracles (oracle/hashcube.py) against what PAPER.md and
textbook routines fix (all CPU, `-m "not gpu"`)."""
from __future__ import annotations

import json
import os

import numpy as np
import pytest

import oracle
from oracle import hashcube as hco
from pins import min_set_1d, sweep_2d

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "flights.json")))
HC_GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "hashcube_fig1b.json")))
FLIGHTS = np.array(GOLD["points"], np.float32)


def tie_heavy(seed, n, d, levels=3):
    rng = np.random.default_rng(seed)
    return rng.integers(0, levels, size=(n, d)).astype(np.float32)


# ------------------------------------------------------------------------------ Fig. 1b / B.1 pins
@pytest.mark.parametrize("impl", ["literal", "vectorised"])
def test_flights_hashcube_fig1b(impl):
    rows = oracle.rows_a(FLIGHTS, with_ext=False)
    if impl == "literal":
        H = hco.hashcube_literal(rows, 3, 4)
        got = [{str(k): v for k, v in h.items()} for h in H]
    else:
        hc = hco.hashcube(rows, 3, 4)
        got = []
        for k in range(hco.n_words(3, 4)):
            h = {}
            for u in range(hc["word_offsets"][k], hc["word_offsets"][k + 1]):
                h[str(int(hc["keys"][u]))] = hc["ids"][hc["key_offsets"][u]:hc["key_offsets"][u + 1]].tolist()
            got.append(h)
    assert got == [HC_GOLD["h0"], HC_GOLD["h1"]]
    # f4 is dominated in every subspace (Fig. 3: B_{f4 notin S} = 1111111) and is stored nowhere
    assert all(4 not in ids for h in got for ids in h.values())


def test_flights_f1_words_L1278():
    """L1278: B_{f1 notin S} is split into w1 = 000 and w0 = 1011 (w = 4)."""
    rows = oracle.rows_b(FLIGHTS)
    H = hco.hashcube_literal(rows, 3, 4)
    key_of = {k: next(key for key, ids in H[k].items() if 1 in ids) for k in range(2)}
    assert format(key_of[0], "04b") == HC_GOLD["f1_w0"] and format(key_of[1], "03b") == HC_GOLD["f1_w1"]


def test_flights_retrieval_example_L1280():
    """S_4 is recorded by h_0 (bit 3): keys with bit 3 unset give {f0} = S_4 of Fig. 1a (reading Q6);
    the keys with bit 3 set (9, 10, 11) hold exactly the complement {f3, f2, f1} of S_4 within the stored
    points."""
    rows = oracle.rows_a(FLIGHTS, with_ext=False)
    hc = hco.hashcube(rows, 3, 4)
    assert hco.query(hc, 3, 4, 4) == GOLD["lattice"]["4"] == [0]
    set_keys = [int(k) for k in hc["keys"][hc["word_offsets"][0]:hc["word_offsets"][1]] if (int(k) >> 3) & 1]
    assert set_keys == [9, 10, 11]
    for delta in range(1, 8):
        assert hco.query(hc, 3, 4, delta) == GOLD["lattice"][str(delta)], delta


# ------------------------------------------------------------------------ reductions / round trips
@pytest.mark.parametrize("seed", range(6))
def test_w1_is_the_lattice(seed):
    """w = 1: every word is one subspace; key 0 (not dominated) lists S_delta exactly, key 1 is never
    stored -- the HashCube degenerates to the lattice of Fig. 1a (computed by Oracle A)."""
    d = 2 + seed % 3
    x = tie_heavy(seed, 9, d)
    rows = oracle.rows_a(x, with_ext=False)
    off, ids = oracle.lattice(rows, d)
    hc = hco.hashcube(rows, d, 1)
    assert (hc["keys"] == 0).all()
    for delta in range(1, 1 << d):
        k = delta - 1
        us = range(hc["word_offsets"][k], hc["word_offsets"][k + 1])
        got = [i for u in us for i in hc["ids"][hc["key_offsets"][u]:hc["key_offsets"][u + 1]].tolist()]
        assert got == ids[off[delta]:off[delta + 1]].tolist(), delta


@pytest.mark.parametrize("w", [1, 2, 3, 4, 5, 7, 8, 16, 31, 32])
@pytest.mark.parametrize("seed", range(4))
def test_retrieval_matches_oracle_a_lattice(w, seed):
    d = [3, 4, 5, 6][seed]
    x = tie_heavy(100 + seed, 14, d)
    rows = oracle.rows_a(x, with_ext=False)
    off, ids = oracle.lattice(rows, d)
    hc = hco.hashcube(rows, d, w)
    for delta in range(1, 1 << d):
        assert hco.query(hc, d, w, delta) == ids[off[delta]:off[delta + 1]].tolist(), (w, delta)


@pytest.mark.parametrize("w", [1, 3, 4, 8, 32])
@pytest.mark.parametrize("seed", range(5))
def test_literal_equals_vectorised(w, seed):
    d = 1 + seed * 2 if seed < 4 else 7
    x = tie_heavy(200 + seed, 12, d)
    rows = oracle.rows_b(x)
    a = hco.to_arrays(hco.hashcube_literal(rows, d, w))
    b = hco.hashcube(rows, d, w)
    for k in a:
        assert np.array_equal(a[k], b[k]), k


def test_compression_invariants():
    """Each point is stored at most once per word (L1276 'at most once per fixed group of w subspaces'),
    and not at all in word k iff it is dominated in every subspace of the word (Oracle A cells)."""
    d, w = 6, 8
    x = tie_heavy(7, 20, d)
    rows = oracle.rows_b(x)
    hc = hco.hashcube(rows, d, w)
    nbits = (1 << d) - 1
    for k in range(hco.n_words(d, w)):
        lo, hi = hc["key_offsets"][hc["word_offsets"][k]], hc["key_offsets"][hc["word_offsets"][k + 1]]
        stored = hc["ids"][lo:hi].tolist()
        assert len(stored) == len(set(stored))
        deltas = [k * w + b + 1 for b in range(w) if k * w + b + 1 <= nbits]
        for p in range(x.shape[0]):
            cells = oracle.cells_a(x, [p] * len(deltas), deltas)
            assert (p in stored) == bool(cells.any()), (k, p)
    n_words = hco.n_words(d, w)
    assert hc["ids"].size <= x.shape[0] * n_words


# ------------------------------------------------------------------------------- partial skycube
def test_partial_flights_levels():
    rows = oracle.rows_a(FLIGHTS, with_ext=False)
    for dp in (1, 2, 3):
        pr = hco.partial_rows(rows, 3, dp)
        off, ids = oracle.lattice(pr, 3)
        for delta in range(1, 8):
            want = GOLD["lattice"][str(delta)] if bin(delta).count("1") <= dp else []
            assert ids[off[delta]:off[delta + 1]].tolist() == want, (dp, delta)


@pytest.mark.parametrize("seed", range(4))
def test_partial_low_levels_textbook(seed):
    """d' = 2: level-1 lists are the argmin sets, level-2 lists the sort-and-sweep skylines (textbook,
    with ties); every higher level is empty."""
    rng = np.random.default_rng(300 + seed)
    n, d = 30, 5
    x = rng.integers(0, 4, size=(n, d)).astype(np.float32)
    pr = hco.partial_rows(oracle.rows_b(x), d, 2)
    off, ids = oracle.lattice(pr, d)
    for delta in range(1, 1 << d):
        got = ids[off[delta]:off[delta + 1]].tolist()
        dims = [i for i in range(d) if (delta >> i) & 1]
        if len(dims) == 1:
            assert got == min_set_1d(x[:, dims[0]])
        elif len(dims) == 2:
            assert got == sweep_2d(x[:, dims[0]], x[:, dims[1]])
        else:
            assert got == []


def test_level_mask_counts():
    from math import comb
    for d in (3, 6, 9):
        for dp in range(0, d + 1):
            m = hco.level_mask_words(d, dp)
            assert sum(bin(int(v)).count("1") for v in m) == sum(comb(d, k) for k in range(1, dp + 1))

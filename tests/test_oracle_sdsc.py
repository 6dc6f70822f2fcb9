"""Pins for the SDSC oracle (Alg. 2, oracle/sdsc.py): the top-down traversal over extended skylines must
reproduce Def. 3 (Oracle A) exactly, ties included (CPU, `-m "not gpu"`)."""
from __future__ import annotations

import itertools
import json
import os

import numpy as np
import pytest

import oracle
from oracle import sdsc

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "flights.json")))


def _members(rows, delta):
    return [p for p in range(rows.shape[0]) if (int(rows[p, delta >> 5]) >> (delta & 31)) & 1]


def test_flights_fig1a_and_line2():
    x = np.array(GOLD["points"], np.float32)
    L, Lp = sdsc.sdsc(x)
    for delta_s, ids in GOLD["lattice"].items():
        assert L[int(delta_s)] == ids
    # Alg. 2 line 2: L+[7] = S+_7 \ S_7 = {f4} (f4 is in S+ yet in no skyline, L104-106)
    assert Lp[7] == [4]
    # S+_3 = {f1, f2, f3, f4} (L104-106): L[3] U L+[3]
    assert sorted(L[3] + Lp[3]) == GOLD["Splus3"]
    off, ids = sdsc.to_lattice(L, 3)
    assert off.tolist() == [0, 0, 1, 2, 5, 6, 9, 12, 16]


def _check_against_def(x):
    n, d = x.shape
    rows, ext = oracle.rows_a(x)
    L, Lp = sdsc.sdsc(x)
    for delta in range(1, 1 << d):
        assert L[delta] == _members(rows, delta), delta
        assert Lp[delta] == sorted(set(_members(ext, delta)) - set(_members(rows, delta))), delta


def test_exhaustive_three_point_sets():
    vals = list(itertools.product([0, 1, 2], repeat=2))
    for combo in itertools.combinations_with_replacement(vals, 3):
        _check_against_def(np.array(combo, np.float32))


@pytest.mark.parametrize("seed", range(25))
def test_random_tie_heavy(seed):
    rng = np.random.default_rng(4000 + seed)
    n, d = int(rng.integers(2, 12)), int(rng.integers(2, 5))
    _check_against_def(rng.integers(0, 3, size=(n, d)).astype(np.float32))


def test_continuous():
    rng = np.random.default_rng(9)
    _check_against_def(rng.random((40, 4)).astype(np.float32))

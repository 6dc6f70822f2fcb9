"""Pins for the CPU oracle against what PAPER.md and mathematics fix (all CPU, `-m "not gpu"`)."""
from __future__ import annotations

import itertools
import json
import os

import numpy as np
import pytest

import datagen
import oracle
from pins import (bit, expected_maxima, expected_maxima_float, fig3_string, members, min_set_1d,
                  sfs_skyline, sfs_strict_skyline, shifted_string, sweep_2d)

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "flights.json")))
FLIGHTS = np.array(GOLD["points"], np.float32)


# ---------------------------------------------------------------- Table 1 / Fig. 1 / Fig. 3 pins
@pytest.mark.parametrize("method", ["a", "b"])
def test_flights_lattice_fig1a(method):
    rows = oracle.rows_a(FLIGHTS, with_ext=False) if method == "a" else oracle.rows_b(FLIGHTS)
    for delta_s, ids in GOLD["lattice"].items():
        assert members(rows, int(delta_s)) == ids, delta_s
    off, ids = oracle.lattice(rows, 3)
    assert off.tolist() == [0, 0, 1, 2, 5, 6, 9, 12, 16]
    assert ids.tolist() == [2, 3, 1, 2, 3, 0, 0, 1, 2, 0, 1, 3, 0, 1, 2, 3]


def test_flights_minutes_same_skycube():
    a = oracle.rows_a(FLIGHTS, with_ext=False)
    b = oracle.rows_a(np.array(GOLD["points_minutes"], np.float32), with_ext=False)
    assert (a == b).all()


def test_flights_shifted_membership_L84():
    rows = oracle.rows_b(FLIGHTS)
    assert shifted_string(rows, 1, 3) == GOLD["shifted_in_S_f1"]


@pytest.mark.parametrize("method", ["a", "b"])
def test_flights_fig3_masks(method):
    if method == "a":
        rows, ext = oracle.rows_a(FLIGHTS)
    else:
        rows, ext = oracle.rows_b(FLIGHTS, with_ext=True)
    for p in range(5):
        assert fig3_string(rows, p, 3, negate=True) == GOLD["fig3_not_in_S"][p], p
        assert fig3_string(ext, p, 3, negate=True) == GOLD["fig3_not_in_Sp"][p], p


def test_flights_extended_skylines_L104():
    rows, ext = oracle.rows_a(FLIGHTS)
    assert members(rows, 3) == GOLD["S3"]
    assert members(ext, 3) == GOLD["Splus3"]
    # L94-96: f3 strictly dominates f4 in 6 (f4 not in S+_6); f3 dominates f4 in 7 but not strictly
    assert not bit(ext, 4, 6) and not bit(rows, 4, 7) and bit(ext, 4, 7)
    # f1 dominates f0 in delta = 3
    assert not bit(rows, 0, 3)
    # Alg. 3 line 2 / Table 1 caption: all five flights are in S+(P), f4 is in no skyline
    assert oracle.ext_full(FLIGHTS).all()
    assert rows[4].sum() == 0


def test_flights_pairwise_masks_L82():
    def mask(a, b, op):
        return "".join("1" if op(a[i], b[i]) else "0" for i in (2, 1, 0))
    f0, f1 = FLIGHTS[0], FLIGHTS[1]
    assert mask(f0, f1, np.less_equal) == GOLD["pairwise"]["f0<=f1"]
    assert mask(f1, f0, np.less_equal) == GOLD["pairwise"]["f1<=f0"]
    assert mask(f0, f1, np.equal) == GOLD["pairwise"]["f0=f1"]


# ---------------------------------------------------------------- exhaustive / brute force
def _a_equals_b(x):
    ra, ea = oracle.rows_a(x)
    rb, eb = oracle.rows_b(x, with_ext=True)
    return (ra == rb).all() and (ea == eb).all()


def test_exhaustive_three_points_3x3_grid():
    vals = list(itertools.product(range(3), repeat=2))
    for trip in itertools.product(vals, repeat=3):
        x = np.array(trip, np.float32)
        assert _a_equals_b(x), trip


def test_exhaustive_four_points_binary_cube():
    vals = list(itertools.product(range(2), repeat=3))
    for quad in itertools.product(vals, repeat=4):
        x = np.array(quad, np.float32)
        assert _a_equals_b(x), quad


@pytest.mark.parametrize("seed", range(40))
def test_random_tie_heavy_a_equals_b(seed):
    rng = np.random.default_rng(1000 + seed)
    n = int(rng.integers(1, 64))
    d = int(rng.integers(1, 7))
    x = datagen.small_int_grid(n, d, int(rng.integers(2, 5)), seed)
    assert _a_equals_b(x)


# ---------------------------------------------------------------- textbook special cases
@pytest.mark.parametrize("seed", range(6))
def test_one_and_two_dim_subspaces_textbook(seed):
    x = datagen.small_int_grid(200, 5, 6, seed) if seed % 2 else datagen.generate("I", 300, 5, seed)
    rows = oracle.rows_b(x)
    d = x.shape[1]
    for i in range(d):
        assert members(rows, 1 << i) == min_set_1d(x[:, i])
    for i, j in itertools.combinations(range(d), 2):
        assert members(rows, (1 << i) | (1 << j)) == sweep_2d(x[:, i], x[:, j])


@pytest.mark.parametrize("dist,seed", [("I", 1), ("A", 2), ("C", 3), ("grid", 4)])
def test_full_space_is_sfs_skyline(dist, seed):
    x = datagen.small_int_grid(300, 4, 5, seed) if dist == "grid" else datagen.generate(dist, 400, 5, seed)
    d = x.shape[1]
    rows = oracle.rows_b(x)
    assert members(rows, (1 << d) - 1) == sfs_skyline(x)
    assert np.nonzero(oracle.ext_full(x))[0].tolist() == sfs_strict_skyline(x)


def test_degenerate_cases():
    # n = 1: in every cuboid
    r = oracle.rows_b(np.array([[0.5, 0.25, 0.75]], np.float32))
    assert r[0, 0] == 0xFE
    # all identical: everyone everywhere (Q9: no dominance when equal on all of delta)
    r = oracle.rows_b(np.ones((7, 4), np.float32))
    assert (r[:, 0] == 0xFFFE).all()
    # chain: only p_0
    r = oracle.rows_b(datagen.chain(9, 3))
    assert r[0, 0] == 0xFE and (r[1:] == 0).all()
    # 2-D antichain (i, n-1-i)
    n = 11
    r = oracle.rows_b(datagen.antichain2d(n))
    assert members(r, 3) == list(range(n))
    assert members(r, 1) == [0] and members(r, 2) == [n - 1]
    # I3 counterexample with ties: (0,1) in S_1 but not in S_3
    r = oracle.rows_b(np.array([[0, 0], [0, 1]], np.float32))
    assert bit(r, 1, 1) and not bit(r, 1, 3)
    # +-inf are ordinary values; -0 == +0
    r = oracle.rows_b(np.array([[-np.inf, 1.0], [0.0, -0.0], [-0.0, 0.0]], np.float32))
    assert members(r, 1) == [0] and members(r, 2) == [1, 2] and members(r, 3) == [0, 1, 2]


def test_nan_is_rejected():
    with pytest.raises(ValueError):
        oracle.rows_b(np.array([[np.nan, 1.0]], np.float32))


# ---------------------------------------------------------------- closed form (statistical)
def test_expected_maxima_closed_form_values():
    # A(1000, k) = 1, 7.49, 28.8, 76.5 ; exact rational recurrence vs float recurrence
    vals = [expected_maxima(1000, k) for k in range(1, 5)]
    assert vals[0] == 1.0
    assert abs(vals[1] - 7.4854708) < 1e-6  # harmonic number H_1000
    for k in range(1, 5):
        assert abs(expected_maxima_float(1000, k) - vals[k - 1]) < 1e-9 * vals[k - 1]


def test_mean_skyline_size_matches_expected_maxima():
    n, d, seeds = 1000, 4, 24
    sums = np.zeros(d + 1)
    cnt = np.zeros(d + 1)
    for s in range(seeds):
        rows = oracle.rows_b(datagen.generate("I", n, d, 500 + s))
        for delta in range(1, 1 << d):
            k = bin(delta).count("1")
            sums[k] += len(members(rows, delta))
            cnt[k] += 1
    for k in range(1, d + 1):
        mean = sums[k] / cnt[k]
        ex = expected_maxima_float(n, k)
        # Var of the number of maxima is O(ex); 3-sigma bound on the mean of cnt[k] samples
        tol = 3.0 * np.sqrt(max(ex, 1.0) / cnt[k]) + 1e-9
        assert abs(mean - ex) <= tol + 0.02 * ex, (k, mean, ex)


# ---------------------------------------------------------------- invariants I1-I8
def _inv_data():
    out = []
    for s in range(3):
        out.append(datagen.small_int_grid(60, 5, 4, 70 + s))
        out.append(datagen.generate("A", 80, 5, 80 + s))
    return out


@pytest.mark.parametrize("k", range(6))
def test_invariants(k):
    x = _inv_data()[k]
    n, d = x.shape
    rows, ext = oracle.rows_b(x, with_ext=True)
    full = (1 << d) - 1
    ext_full = oracle.ext_full(x)
    for p in range(n):
        if not ext_full[p]:
            assert rows[p].sum() == 0                                          # I1
        for delta in range(1, full + 1):
            if bit(rows, p, delta):
                assert bit(ext, p, delta)                                       # S_delta subset of S+_delta
            if not bit(ext, p, delta):
                sub = (delta - 1) & delta
                while sub:
                    assert not bit(ext, p, sub)                                 # I2 downward closed
                    sub = (sub - 1) & delta
    assert all(len(members(rows, delta)) >= 1 for delta in range(1, full + 1))   # I4
    rng = np.random.default_rng(k)
    perm = rng.permutation(n)
    rp = oracle.rows_b(x[perm])
    assert (rp == rows[perm]).all()                                             # I5
    cperm = rng.permutation(d)
    rc = oracle.rows_b(np.ascontiguousarray(x[:, cperm]))
    for delta in range(1, full + 1):                                            # I6
        mapped = sum(1 << int(np.nonzero(cperm == i)[0][0]) for i in range(d) if delta >> i & 1)
        assert members(rc, mapped) == members(rows, delta)
    # I7: strictly increasing per-dimension maps (rank transform: exact in float32)
    xr = np.empty_like(x)
    for i in range(d):
        u, inv = np.unique(x[:, i], return_inverse=True)
        xr[:, i] = (inv * 3 + 1).astype(np.float32)
    assert (oracle.rows_b(xr) == rows).all()
    # I8: duplicating a row
    xd = np.concatenate([x, x[3:4]], axis=0)
    rd = oracle.rows_b(xd)
    assert (rd[:n] == rows).all() and (rd[n] == rows[3]).all()


def test_distinct_values_upward_closed():
    x = datagen.distinct_columns(120, 5, 9)
    rows, ext = oracle.rows_b(x, with_ext=True)
    assert (rows == ext).all()                                                  # I3: S = S+
    full = 31
    for p in range(x.shape[0]):
        for delta in range(1, full + 1):
            if bit(rows, p, delta):
                for j in range(5):
                    assert bit(rows, p, delta | (1 << j))                       # S_d' subset S_d


def test_cells_agree_with_rows():
    x = datagen.small_int_grid(90, 6, 4, 3)
    rows = oracle.rows_b(x)
    rng = np.random.default_rng(0)
    pids = rng.integers(0, 90, 500)
    deltas = rng.integers(1, 64, 500).astype(np.uint32)
    cells = oracle.cells_a(x, pids, deltas)
    for k in range(500):
        assert cells[k] == bit(rows, pids[k], int(deltas[k]))


def test_rows_b_point_subset():
    x = datagen.generate("A", 500, 6, 11)
    rows = oracle.rows_b(x)
    pids = np.array([0, 17, 499, 250], np.int64)
    assert (oracle.rows_b(x, pids) == rows[pids]).all()

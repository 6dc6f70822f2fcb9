"""Independent textbook routines and paper conversions used to PIN the oracle (not the oracle itself).

Each routine computes something the paper or textbook mathematics fixes by a different algorithm
than the oracle's literal Def. 1-3 loop, so that a plausible oracle mistake (a dropped term, a
flipped comparison, a transposed operand) fails at least one of them.
"""
from __future__ import annotations

from fractions import Fraction

import numpy as np


def bit(rows, p, delta):
    return bool((int(rows[p, delta >> 5]) >> (delta & 31)) & 1)


def members(rows, delta):
    return [p for p in range(rows.shape[0]) if bit(rows, p, delta)]


def level_order(d):
    """Lattice-level order of subspaces (Fig. 3, reading Q2): by (popcount, value)."""
    return sorted(range(1, 1 << d), key=lambda s: (bin(s).count("1"), s))


def fig3_string(rows, p, d, negate):
    """Render the paper's Fig. 3 string for point p: rightmost char = first subspace in level order."""
    chars = []
    for delta in level_order(d):
        b = bit(rows, p, delta)
        chars.append("1" if (not b if negate else b) else "0")
    return "".join(reversed(chars))


def shifted_string(rows, p, d):
    """The paper's B_{p in S} (L84): bit delta-1, most significant (delta = 2^d - 1) first."""
    return "".join("1" if bit(rows, p, delta) else "0" for delta in range((1 << d) - 1, 0, -1))


def min_set_1d(col):
    """pc(delta) = 1: the skyline is every point attaining the minimum (ties included)."""
    m = col.min()
    return sorted(np.nonzero(col == m)[0].tolist())


def sweep_2d(x, y):
    """pc(delta) = 2 by sort-and-sweep (textbook), with exact tie handling.

    Sort by x; for each distinct x value v, a point with y-value t is in the skyline iff
    t is the minimum y among points with x == v AND t is strictly below every y seen at x < v.
    """
    order = np.lexsort((y, x))
    out = []
    best_prev = np.inf
    i = 0
    n = len(order)
    while i < n:
        j = i
        v = x[order[i]]
        while j < n and x[order[j]] == v:
            j += 1
        grp = order[i:j]
        m = y[grp].min()
        if m < best_prev:
            out.extend(int(k) for k in grp if y[k] == m)
        best_prev = min(best_prev, m)
        i = j
    return sorted(out)


def sfs_skyline(pts):
    """Full-space skyline by Sort-Filter-Skyline (Chomicki et al.), a different algorithm from Def. 2.

    Points are visited in ascending coordinate-sum order; a point is in the skyline iff no point in
    the window dominates it.  Equal-sum points cannot dominate each other unless identical (and
    identical points never dominate), so visiting order within equal sums does not matter.
    """
    n = pts.shape[0]
    sums = pts.astype(np.float64).sum(axis=1)
    order = np.argsort(sums, kind="stable")
    window = []
    res = []
    for k in order:
        p = pts[k]
        dominated = False
        for w in window:
            q = pts[w]
            if np.all(q <= p) and np.any(q < p):
                dominated = True
                break
        if not dominated:
            window.append(k)
            res.append(int(k))
    return sorted(res)


def sfs_strict_skyline(pts):
    """Full-space extended skyline S+ (strict dominance only) by the same windowed scan.

    Window = every point seen so far (strict dominance is not transitive through equal points,
    so no pruning of the window); ordering by sum still guarantees dominators come first.
    """
    sums = pts.astype(np.float64).sum(axis=1)
    order = np.argsort(sums, kind="stable")
    seen = []
    res = []
    for k in order:
        p = pts[k]
        if not any(np.all(pts[w] < p) for w in seen):
            res.append(int(k))
        seen.append(k)
    return sorted(res)


def expected_maxima(n: int, k: int) -> float:
    """Expected number of maxima of n i.i.d. continuous points in k dimensions (Bentley et al.):
    A(n,1) = 1, A(n,k) = sum_{i=1..n} A(i,k-1)/i.  Exact rationals, then float."""
    prev = [Fraction(1)] * (n + 1)  # A(i, 1) = 1
    for _ in range(2, k + 1):
        cur = [Fraction(0)] * (n + 1)
        acc = Fraction(0)
        for i in range(1, n + 1):
            acc += prev[i] / i
            cur[i] = acc
        prev = cur
    return float(prev[n])


def expected_maxima_float(n: int, k: int) -> float:
    prev = np.ones(n + 1)
    for _ in range(2, k + 1):
        cur = np.zeros(n + 1)
        cur[1:] = np.cumsum(prev[1:] / np.arange(1, n + 1))
        prev = cur
    return float(prev[n])

"""Randomised parity sweep: many small seeded datasets of every shape class (random d, n, value
distribution, tie level, duplicated rows, +-0 / +-inf, forced K3 design and state mode, partial levels,
HashCube word lengths), each compared bit for bit with the CPU oracle.  Needs a B200."""
from __future__ import annotations

import numpy as np
import pytest

import datagen
import oracle
from oracle import hashcube as hco
import paper_conf_sigmod_boghcsa17_b200 as sky

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    sky.lib()


def _dataset(rng):
    d = int(rng.integers(1, 17))
    n = int(rng.integers(1, 2500 if d <= 12 else 700))
    kind = rng.integers(0, 6)
    if kind == 0:
        x = rng.integers(0, int(rng.integers(2, 6)), size=(n, d)).astype(np.float32)  # heavy ties
    elif kind == 1:
        x = datagen.generate("A", n, d, int(rng.integers(1 << 30)))
    elif kind == 2:
        x = datagen.generate("I", n, d, int(rng.integers(1 << 30)))
    elif kind == 3:
        x = datagen.generate("C", n, d, int(rng.integers(1 << 30)))
    elif kind == 4:
        x = datagen.generate("ct", n, d, int(rng.integers(1 << 30)))
    else:  # special values and duplicated rows
        x = rng.choice(np.array([-np.inf, -1.0, -0.0, 0.0, 0.5, 1.0, np.inf], np.float32), size=(n, d))
    if n > 3 and rng.random() < 0.3:
        x[rng.integers(0, n, n // 4)] = x[rng.integers(0, n, n // 4)]  # duplicate rows
    return np.ascontiguousarray(x, dtype=np.float32)


@pytest.mark.parametrize("seed", range(300))
def test_random_case(tuning, seed):
    rng = np.random.default_rng(10_000 + seed)
    x = _dataset(rng)
    n, d = x.shape
    design = ["", "A", "O"][int(rng.integers(0, 3))]
    mode = ["", "0", "1", "2"][int(rng.integers(0, 4))]
    if design:
        tuning("k3_design", design)
    if mode:
        tuning("k3_mode", int(mode))
    want = oracle.rows_b(x)
    level = int(rng.integers(0, d + 1)) if rng.random() < 0.3 else 0
    r = sky.skycube_build(x, max_level=level)
    exp = hco.partial_rows(want, d, level) if level else want
    bad = np.nonzero((r["rows"] != exp).any(axis=1))[0]
    assert bad.size == 0, f"n={n} d={d} design={design} mode={mode} level={level}: rows {bad[:5]}"
    off, ids = oracle.lattice(exp, d)
    assert np.array_equal(r["offsets"], off) and np.array_equal(r["ids"], ids)
    assert np.array_equal(r["ext_ids"], np.nonzero(oracle.ext_full(x))[0])
    if d <= 14:
        w = int(rng.choice([1, 3, 8, 32]))
        got = sky.skycube_build_hashcube(x, w, max_level=level)
        want_hc = hco.hashcube(exp, d, w)
        for k in ("word_offsets", "keys", "key_offsets", "ids"):
            assert np.array_equal(got[k], want_hc[k]), (k, w)

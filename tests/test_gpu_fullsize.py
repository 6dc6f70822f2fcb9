"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times (pipeline.DeviceSkycube),
on outputs the oracle can compute one by one (seeded samples of points), plus properties that hold at
any size.  Needs a B200."""
from __future__ import annotations

import numpy as np
import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu

SAMPLE = 48


@pytest.fixture(scope="module")
def engine():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_sigmod_boghcsa17_b200.pipeline import DeviceSkycube
    eng = DeviceSkycube(0)
    yield eng
    eng.close()


def _build(engine, x):
    import torch
    pts = torch.from_numpy(x).cuda()
    out = engine.build(pts, lists=True, membership=True)
    torch.cuda.synchronize()
    return out


def _rows_of(out, pids):
    import torch
    mem = out["membership"]
    return mem[torch.as_tensor(pids, device=mem.device)].cpu().numpy().view(np.uint32)


@pytest.mark.parametrize("name", ["C2", "C3C", "C3I", "C3A", "C5", "H", "C4"])
def test_full_size_sampled_rows_and_lattice_properties(engine, name):
    import torch
    cfg = datagen.config(name)
    x = cfg.data()
    n, d = x.shape
    out = _build(engine, x)
    m = out["n_ext"]
    rng = np.random.default_rng(1234)
    ext_ids = out["ext_ids"].cpu().numpy()
    assert np.all(np.diff(ext_ids) > 0) and len(ext_ids) == m
    # half the sample from S+ (interesting rows), half uniform (mostly zero rows outside S+)
    pids = np.unique(np.concatenate([rng.choice(ext_ids, SAMPLE // 2, replace=False),
                                     rng.choice(n, SAMPLE // 2, replace=False)]))
    want_rows, want_ext = oracle.rows_b(x, pids, with_ext=True)
    got = _rows_of(out, pids)
    bad = np.nonzero((got != want_rows).any(axis=1))[0]
    assert bad.size == 0, f"{name}: rows of points {pids[bad][:5]} differ"
    full = (1 << d) - 1
    in_ext = ((want_ext[:, full >> 5] >> (full & 31)) & 1).astype(bool)
    assert np.array_equal(np.isin(pids, ext_ids), in_ext), f"{name}: S+ membership differs on the sample"

    # lattice properties at full size
    off = out["offsets"].cpu().numpy()
    nsub = 1 << d
    assert off[0] == 0 and off[1] == 0 and np.all(np.diff(off) >= 0)
    assert np.all(np.diff(off)[1:] >= 1), "I4: every subspace skyline is non-empty"
    mem = out["membership"]
    pop = sum(int(((mem >> b) & 1).sum(dtype=torch.int64).item()) for b in range(32))
    assert pop == off[-1], "total ids == total membership bits"
    ids = out["ids"]
    deltas = sorted(set([1, 2, nsub - 1, nsub // 2 + 1] + rng.integers(1, nsub, 6).tolist()))
    for delta in deltas:
        lst = ids[off[delta]:off[delta + 1]].cpu().numpy()
        assert np.all(np.diff(lst) > 0), f"ids ascending in delta {delta}"
        word = mem[:, delta >> 5].cpu().numpy().view(np.uint32)
        members = np.nonzero((word >> (delta & 31)) & 1)[0]
        assert np.array_equal(lst, members), f"lattice of delta {delta} == transpose of rows"
    # I1: rows outside S+ are zero
    nz = torch.nonzero(mem.any(dim=1)).flatten().cpu().numpy()
    assert np.all(np.isin(nz, ext_ids))


def test_c2_full_oracle(engine):
    x = datagen.config("C2").data()
    out = _build(engine, x)
    want = oracle.rows_b(x)
    got = out["membership"].cpu().numpy().view(np.uint32)
    assert np.array_equal(got, want)
    offs, ids = oracle.lattice(want, x.shape[1])
    assert np.array_equal(out["offsets"].cpu().numpy(), offs)
    assert np.array_equal(out["ids"].cpu().numpy(), ids)


@pytest.mark.parametrize("name", ["C3A", "C5", "H"])
def test_full_size_hashcube_sampled(engine, name):
    """HashCube (K5, w = 32) at full size through the bench launch path: for seeded sample points the oracle
    row (Oracle B) fixes, word by word, the key the point must be stored under (or that it is absent); plus
    properties: keys ascending per word, ids ascending per key, each point at most once per word, and the
    number of stored ids = the number of not-all-dominated (point, word) pairs of the GPU's own rows."""
    import torch
    from oracle import hashcube as hco
    cfg = datagen.config(name)
    x = cfg.data()
    n, d = x.shape
    out = engine.build(torch.from_numpy(x).cuda(), lists=False, membership=True, hashcube_w=32)
    torch.cuda.synchronize()
    hc = {k: v.cpu().numpy() for k, v in out["hashcube"].items()}
    keys = hc["keys"].view(np.uint32)
    woff, koff, ids = hc["word_offsets"], hc["key_offsets"], hc["ids"]
    nw = hco.n_words(d, 32)
    assert woff.shape[0] == nw + 1 and woff[0] == 0 and woff[-1] == keys.size and koff[-1] == ids.size
    key_word = np.repeat(np.arange(nw), np.diff(woff))
    assert np.all((np.diff(keys.astype(np.int64)) > 0) | (np.diff(key_word) > 0)), "keys ascending per word"
    id_key = np.repeat(np.arange(keys.size), np.diff(koff))
    assert np.all((np.diff(ids) > 0) | (np.diff(id_key) > 0)), "ids ascending per key"
    # where every point is stored, per word: (word, id) -> key
    id_word = key_word[id_key]
    pair = id_word.astype(np.int64) * n + ids
    assert np.unique(pair).size == pair.size, "each point at most once per word"
    ext_ids = out["ext_ids"].cpu().numpy()
    rng = np.random.default_rng(77)
    pids = np.unique(np.concatenate([rng.choice(ext_ids, 16, replace=False), rng.choice(n, 8, replace=False)]))
    want = hco.hashcube(oracle.rows_b(x, pids), d, 32)  # HashCube of the sample alone (ids 0..len-1)
    order = np.argsort(pair, kind="stable")
    sp = pair[order]
    for s, p in enumerate(pids):
        for k in range(nw):
            # oracle: key of sample point s in word k, or absent
            lo, hi = want["word_offsets"][k], want["word_offsets"][k + 1]
            wkey = None
            for u in range(lo, hi):
                if s in want["ids"][want["key_offsets"][u]:want["key_offsets"][u + 1]]:
                    wkey = int(want["keys"][u])
            j = np.searchsorted(sp, k * n + p)
            found = j < sp.size and sp[j] == k * n + p
            gkey = int(keys[id_key[order[j]]]) if found else None
            assert gkey == wkey, f"{name}: point {p} word {k}: gpu {gkey} oracle {wkey}"
    # stored ids == (point, word) pairs of the rows whose word is not all dominated
    notS = ~out["membership"].cpu().numpy().view(np.uint32)
    W = notS.shape[1]
    stored = 0
    for k in range(nw):
        v = (notS[:, k].astype(np.uint64) >> np.uint64(1))
        if k + 1 < W:
            v |= (notS[:, k + 1].astype(np.uint64) & np.uint64(1)) << np.uint64(31)
        valid = min(32, (1 << d) - 1 - 32 * k)
        full = np.uint64((1 << valid) - 1)
        stored += int(np.count_nonzero((v & full) != full))
    assert stored == ids.size

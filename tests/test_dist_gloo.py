"""Multi-rank sharding and exchange logic of pipeline.py on CPU (gloo, world_size 2 and 3).

The per-rank kernel outputs are stood in by the CPU oracle (test infrastructure), computed for exactly the
ranges the GPU path gives each rank; the real exchange code (pipeline.exchange_ext / exchange_totals /
gather_rows) then has to make the distributed result the single-rank answer:
  * the S+ flags every rank installs equal the full S+ (exchange_ext);
  * the task ranges tile S+ in rank order, so each subspace's global list is the rank-major concatenation of
    the ranks' lists and a rank's segment of subspace delta starts at offsets[delta] + the counts of the
    ranks before it (the placement the lattice scatter kernel performs, from the gathered totals);
  * the id slices tile [0, n), so every membership row is written by exactly one rank;
  * gather_rows reassembles the tiled row buffer the HashCube needs.
"""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import datagen
import oracle
from paper_conf_sigmod_boghcsa17_b200 import pipeline as pl
from paper_conf_sigmod_boghcsa17_b200 import words_per_row


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _key_order(x):
    # Λ2 ordering stand-in (test side): sort by the sum of order-preserving keys, stable by id
    b = x.view(np.uint32).astype(np.uint64)
    b = np.where((b & 0x7fffffff) == 0, 0, b)
    o = np.where(b & 0x80000000, (~b) & 0xffffffff, b | 0x80000000)
    return np.argsort(o.sum(axis=1), kind="stable")


def _tiled(rows_by_j, m, d, nwords):
    W = words_per_row(d)
    out = np.zeros(nwords, np.uint32)
    for j in range(m):
        g, l = divmod(j, 32)
        out[g * W * 32 + np.arange(W) * 32 + l] = rows_by_j[j]
    return out


def _counts(rows, d):
    """Per-subspace member counts of a set of membership rows."""
    nsub = 1 << d
    bits = np.zeros(nsub, np.int64)
    for delta in range(1, nsub):
        bits[delta] = int(((rows[:, delta >> 5] >> np.uint32(delta & 31)) & 1).sum())
    return bits


def _worker(rank, world, port, x, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        n, d = x.shape
        nsub = 1 << d
        order = _key_order(x)
        ext_full = oracle.ext_full(x)
        # --- K1 stand-in: this rank's blocks of sorted positions
        ext8 = torch.zeros(n, dtype=torch.uint8)
        off, step = pl.prefilter_assignment(rank, world)
        nblk = (n + pl.PREFILTER_BLOCK - 1) // pl.PREFILTER_BLOCK
        for t in range(off, nblk, step):
            for s in range(t * pl.PREFILTER_BLOCK, min(n, (t + 1) * pl.PREFILTER_BLOCK)):
                ext8[s] = int(ext_full[order[s]])
        pl.exchange_ext(ext8)
        flags_sorted = ext8.numpy().astype(bool)
        ext_ids = np.sort(order[flags_sorted])
        m = len(ext_ids)
        # --- K3 stand-in: the rows of this rank's task range, in the tiled layout
        rows = oracle.rows_b(x)
        j0, j1 = pl.task_range(m, world, rank)
        nwords = pl.rows_buffer_words(m, d)
        mine = np.zeros((m, words_per_row(d)), np.uint32)
        mine[j0:j1] = rows[ext_ids[j0:j1]]
        rows32 = torch.from_numpy(_tiled(mine, m, d, nwords).view(np.int32).copy())
        # --- K4 count stand-in: this rank's per-subspace totals; the real exchange gathers them
        totals = torch.from_numpy(_counts(rows[ext_ids[j0:j1]], d))
        all_totals = pl.exchange_totals(totals).numpy().reshape(world, nsub)
        # --- HashCube path: reassemble the tiled rows
        pl.gather_rows(rows32, m, d)
        q.put((rank, ext_ids, (j0, j1), all_totals, rows32.numpy().view(np.uint32).copy(),
               pl.id_slice(n, world, rank)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,dist_name,n,d", [(2, "A", 4500, 5), (3, "A", 7000, 3), (2, "grid", 4200, 6)])
def test_sharded_exchange_reassembles_single_rank_result(world, dist_name, n, d):
    x = datagen.small_int_grid(n, d, 4, 3) if dist_name == "grid" else datagen.generate(dist_name, n, d, 17)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, x, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    res.sort(key=lambda t: t[0])
    nsub = 1 << d
    rows = oracle.rows_b(x)
    ext_ids = np.nonzero(oracle.ext_full(x))[0]
    m = len(ext_ids)
    off, ids = oracle.lattice(rows, d)
    # S+ agreed on every rank; task ranges tile [0, m) in rank order; id slices tile [0, n)
    ranges = [r[2] for r in res]
    assert ranges[0][0] == 0 and ranges[-1][1] == m
    assert all(ranges[i][1] == ranges[i + 1][0] for i in range(world - 1))
    slices = [r[5] for r in res]
    assert slices[0][0] == 0 and slices[-1][1] == n and all(slices[i][1] == slices[i + 1][0] for i in range(world - 1))
    for rank, eids, _, all_totals, rows32, _ in res:
        assert np.array_equal(eids, ext_ids)
        # gathered totals: rank-major, and their sum is the global count of every subspace
        assert np.array_equal(all_totals.sum(axis=0)[1:], np.diff(off)[1:])
        # the placement: rank r's ids of delta are the global list's slice after the earlier ranks' counts
        for delta in range(1, nsub):
            lst = ids[off[delta]:off[delta + 1]]
            pos = off[delta]
            for r in range(world):
                a, b = ranges[r]
                seg = ids[pos:pos + all_totals[r, delta]]
                want = np.array([p for p in ext_ids[a:b] if (rows[p, delta >> 5] >> (delta & 31)) & 1], np.int32)
                assert np.array_equal(seg, want), (rank, r, delta)
                pos += all_totals[r, delta]
            assert pos == off[delta + 1] and np.all(np.diff(lst) > 0)
        # the HashCube path's row gather reassembles the full tiled buffer
        assert np.array_equal(rows32, _tiled(rows[ext_ids], m, d, pl.rows_buffer_words(m, d))), rank


def test_sharding_arithmetic():
    for m in [0, 1, 31, 32, 33, 1000, 123457]:
        for world in [1, 2, 3, 8]:
            rs = [pl.task_range(m, world, r) for r in range(world)]
            assert sum(b - a for a, b in rs) == m
            assert rs[0][0] == 0 and rs[-1][1] == m
            for i, (a, b) in enumerate(rs):
                assert a <= b and (a % 32 == 0 or a == b == m)
                if i:
                    assert rs[i - 1][1] == a
            groups = [(b - a + 31) // 32 for a, b in rs]
            assert max(groups) - min(groups) <= 1 or m == 0
    for n in [0, 1, 7, 1000, 581012]:
        for world in [1, 2, 3, 8]:
            sl = [pl.id_slice(n, world, r) for r in range(world)]
            assert sl[0][0] == 0 and sl[-1][1] == n and all(sl[i][1] == sl[i + 1][0] for i in range(world - 1))


def _codes_worker(rank, world, port, codes, R, mino, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        d, n = codes.shape
        b, e = pl.dim_slice(d, world, rank)
        per = -(-d // world)
        # K2 stand-in: this rank's slice of the dimension-major codes, counts and minimum keys (zero elsewhere)
        mine = torch.zeros((per, n), dtype=torch.int16)
        mine[: e - b] = torch.from_numpy(codes[b:e].astype(np.int16))
        Rl = torch.zeros(d, dtype=torch.int64)
        ml = torch.zeros(d, dtype=torch.int64)
        Rl[b:e] = torch.from_numpy(R[b:e].astype(np.int64))
        ml[b:e] = torch.from_numpy(mino[b:e].astype(np.int64))
        allc, Ra, ma = pl.exchange_codes(mine, Rl, ml, d)
        q.put((rank, allc.numpy().view(np.uint16).copy(), Ra.numpy().view(np.uint32).copy(),
               ma.numpy().view(np.uint32).copy()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,d", [(2, 12), (3, 12), (3, 2), (2, 16), (8, 3)])
def test_codes_exchange_reassembles_all_dimensions(world, d):
    """The sharded prepare (pipeline.exchange_codes): every rank computes the codes of its slice of the
    dimensions; after the all-gather every rank holds the codes of every dimension in dimension order, and the
    per-dimension counts / minimum keys (uint32, including values above 2^31) of every dimension."""
    rng = np.random.default_rng(5 + d)
    n = 1500
    codes = rng.integers(0, 32768, size=(d, n)).astype(np.uint16)
    R = rng.integers(1, 2 ** 32, size=d, dtype=np.uint64).astype(np.uint32)
    mino = rng.integers(0, 2 ** 32, size=d, dtype=np.uint64).astype(np.uint32)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_codes_worker, args=(r, world, port, codes, R, mino, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    sl = [pl.dim_slice(d, world, r) for r in range(world)]
    assert sl[0][0] == 0 and sl[-1][1] == d and all(sl[i][1] == sl[i + 1][0] for i in range(world - 1))
    for rank, allc, Ra, ma in res:
        assert np.array_equal(allc, codes), rank
        assert np.array_equal(Ra, R) and np.array_equal(ma, mino), rank

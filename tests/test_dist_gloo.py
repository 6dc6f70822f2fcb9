"""Multi-rank sharding and exchange logic of pipeline.py on CPU (gloo, world_size 2 and 3).

The per-rank kernel outputs are stood in by the CPU oracle (test infrastructure), written into exactly
the buffers and ranges the GPU path writes; the real exchange code (pipeline.exchange_ext /
exchange_rows) then has to reassemble the full single-rank answer byte for byte.
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


def _worker(rank, world, port, x, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        n, d = x.shape
        order = _key_order(x)
        ext_full = oracle.ext_full(x)
        # --- K1 stand-in: this rank's tiles of sorted positions
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
        # --- K3 stand-in: rows of this rank's task range, tiled layout, global offsets
        rows = oracle.rows_b(x)
        nwords = pl.rows_buffer_words(m, d, world)
        buf = np.zeros(nwords, np.uint32)
        j0, j1 = pl.task_range(m, world, rank)
        assert j0 % 32 == 0 or j0 == j1
        part = _tiled(np.where(np.arange(m)[:, None] >= j0, rows[ext_ids], 0) * (np.arange(m)[:, None] < j1),
                      m, d, nwords)
        buf[:] = part
        rows32 = torch.from_numpy(buf.view(np.int32).copy())
        pl.exchange_rows(rows32, m, d)
        q.put((rank, flags_sorted, ext_ids, rows32.numpy().view(np.uint32).copy(), (j0, j1)))
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
    # single-rank reference: full oracle rows in the tiled layout
    rows = oracle.rows_b(x)
    ext_ids = np.nonzero(oracle.ext_full(x))[0]
    m = len(ext_ids)
    want = _tiled(rows[ext_ids], m, d, pl.rows_buffer_words(m, d, world))
    ranges = [r[4] for r in res]
    assert ranges[0][0] == 0 and ranges[-1][1] == m
    assert all(ranges[i][1] == ranges[i + 1][0] for i in range(world - 1))
    for rank, flags, eids, rows32, _ in res:
        assert np.array_equal(eids, ext_ids)
        assert np.array_equal(rows32, want), rank


def test_sharding_arithmetic():
    for m in [0, 1, 31, 32, 33, 1000, 123457]:
        for world in [1, 2, 3, 8]:
            rs = [pl.task_range(m, world, r) for r in range(world)]
            covered = sum(b - a for a, b in rs)
            assert covered == m
            for a, b in rs:
                assert a <= b and (a % 32 == 0 or a == b == m)
            if m:
                assert pl.chunk_words(m, 12, world) * world <= pl.rows_buffer_words(m, 12, world)

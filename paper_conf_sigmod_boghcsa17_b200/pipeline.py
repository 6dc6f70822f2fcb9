"""Per-rank device pipeline of the MDMC skycube, one process per GPU (torch.distributed for plumbing).

Sharding (the paper's device-level data parallelism of MDMC, L308-310, L420 "every
task is independent, there is no need for synchronisation"):

  1. prepare                                     K0 on every rank; K2 (per-dimension sort -> dense-rank codes) on
                                                  the rank's slice of the dimensions (dim_slice), all_gather of the
                                                  codes (world x ceil(d/world) x n uint16: 24 MB at H) and of the
                                                  per-dimension counts; the static-tree order replicated
  2. K1 prefilter                                 blocks of 512 static-tree positions, block b on rank b % world
  3. exchange S+ flags                            all_reduce(MAX) of a uint8 flag vector (NCCL over NVLink)
  4. install S+ (replicated)
  5. K3 MDMC                                      contiguous ranges of 32-point groups of S+, split evenly
  6. K4 compaction, sharded                       each rank: membership rows of its own tasks by id (plus zero
                                                  rows for the points outside S+ in its slice of ids) and the
                                                  per-subspace counts of its rows; all_gather of the counts
                                                  (world x 2^d int64); each rank places its ids at their
                                                  global positions of the lattice and writes them
  7. HashCube (optional)                          needs every row: all_gather of the rows, then K5 on each rank

No row, membership or lattice data crosses between ranks on the lattice path: the result is distributed, each
rank holding the rows of its tasks and its segments of every subspace list at their global positions (a
caller assembles one array by letting every rank write into one shared/pinned buffer, as the C-ABI's
single-process num_gpus path does).  The collective helpers are plain torch.distributed calls so that the
same code runs on NCCL (GPU) and gloo (CPU tests).  Only the kernels are native; nothing here computes
skycube values.
"""
from __future__ import annotations

from dataclasses import dataclass

import torch
import torch.distributed as dist

from . import Context, words_per_row

PREFILTER_BLOCK = 512  # tree positions per K1 CTA (k1_prefilter.cu kTasks)
GROUP = 32


# ------------------------------------------------------------------ pure sharding arithmetic
def prefilter_assignment(rank: int, world: int):
    """(block_offset, block_step) of the K1 blocks a rank processes."""
    return rank, world


def dim_slice(d: int, world: int, rank: int):
    """[dim_begin, dim_end) of the dimensions whose codes (K2) a rank computes in the sharded prepare."""
    per = -(-d // world)
    return min(d, rank * per), min(d, (rank + 1) * per)


def task_range(m: int, world: int, rank: int):
    """[j_begin, j_end) of the S+ tasks of a rank: the 32-task groups split as evenly as possible, in rank order
    (the same split as capi.cu shard_range)."""
    groups = (m + GROUP - 1) // GROUP
    g0, g1 = groups * rank // world, groups * (rank + 1) // world
    return min(m, g0 * GROUP), min(m, g1 * GROUP)


def id_slice(n: int, world: int, rank: int):
    """[lo, hi) of the point ids whose non-S+ membership rows a rank zeroes."""
    return n * rank // world, n * (rank + 1) // world


def rows_buffer_words(m: int, d: int) -> int:
    return max(1, (m + GROUP - 1) // GROUP) * GROUP * words_per_row(d)


# ------------------------------------------------------------------ collectives (NCCL or gloo)
def _staged(t: torch.Tensor, group) -> bool:
    """gloo does not run every collective on CUDA tensors: stage through host memory there (used by the
    single-GPU multi-rank tests; NCCL never stages)."""
    return t.is_cuda and dist.get_backend(group) == "gloo"


def _world(group):
    return dist.get_world_size(group) if dist.is_initialized() else 1


def exchange_ext(ext8: torch.Tensor, group=None):
    """Combine per-rank S+ flags: every position was written by exactly one rank, others are 0."""
    if _world(group) > 1:
        if _staged(ext8, group):
            h = ext8.cpu()
            dist.all_reduce(h, op=dist.ReduceOp.MAX, group=group)
            ext8.copy_(h)
        else:
            dist.all_reduce(ext8, op=dist.ReduceOp.MAX, group=group)
    return ext8


def exchange_totals(totals: torch.Tensor, group=None) -> torch.Tensor:
    """All-gather every rank's per-subspace counts: [world * 2^d] int64, rank-major."""
    world = _world(group)
    if world == 1:
        return totals
    out = torch.empty(world * totals.numel(), dtype=totals.dtype, device=totals.device)
    if _staged(totals, group):
        h = torch.empty(world * totals.numel(), dtype=totals.dtype)
        dist.all_gather_into_tensor(h, totals.cpu(), group=group)
        out.copy_(h)
    else:
        dist.all_gather_into_tensor(out, totals, group=group)
    return out


def exchange_codes(mine: torch.Tensor, R: torch.Tensor, minord: torch.Tensor, d: int, group=None):
    """All-gather the ranks' dimension slices of the codes (each rank [ceil(d/world), n] uint16 as int16, the
    rows past its slice unused) into [d, n], and combine the per-dimension distinct counts and minimum keys
    (uint32 [d] as int64, each entry written by exactly one rank, zero elsewhere: a SUM)."""
    world = _world(group)
    per, n = mine.shape
    mb = mine.contiguous().view(torch.uint8)  # 16-bit codes travel as bytes (neither gloo nor NCCL reduce int16)
    if _staged(mine, group):
        h = torch.empty((world * per, 2 * n), dtype=torch.uint8)
        dist.all_gather_into_tensor(h, mb.cpu(), group=group)
        allc = h.to(mine.device)
        rm = torch.stack([R, minord]).cpu()
        dist.all_reduce(rm, op=dist.ReduceOp.SUM, group=group)
        rm = rm.to(mine.device)
    else:
        allc = torch.empty((world * per, 2 * n), dtype=torch.uint8, device=mine.device)
        dist.all_gather_into_tensor(allc, mb, group=group)
        rm = torch.stack([R, minord])
        dist.all_reduce(rm, op=dist.ReduceOp.SUM, group=group)
    allc = allc.view(mine.dtype)
    rows = [allc[r * per: r * per + (dim_slice(d, world, r)[1] - dim_slice(d, world, r)[0])] for r in range(world)]
    return torch.cat(rows).contiguous(), rm[0].to(torch.int32).contiguous(), rm[1].to(torch.int32).contiguous()


def gather_rows(rows32: torch.Tensor, m: int, d: int, group=None):
    """Assemble every rank's row range into the full tiled row buffer (HashCube output only): ranges are
    contiguous but unequal, so each rank contributes a padded chunk of the largest range."""
    world = _world(group)
    if world == 1:
        return rows32
    rank = dist.get_rank(group)
    W = words_per_row(d)
    gw = GROUP * W
    ranges = [task_range(m, world, r) for r in range(world)]
    cmax = max((b - a + GROUP - 1) // GROUP for a, b in ranges) * gw
    j0, j1 = ranges[rank]
    mine = torch.zeros(max(cmax, 1), dtype=rows32.dtype, device=rows32.device)
    nw = (j1 - j0 + GROUP - 1) // GROUP * gw
    mine[:nw] = rows32[j0 // GROUP * gw: j0 // GROUP * gw + nw]
    if _staged(rows32, group):
        h = torch.empty(world * mine.numel(), dtype=rows32.dtype)
        dist.all_gather_into_tensor(h, mine.cpu(), group=group)
        allc = h.to(rows32.device)
    else:
        allc = torch.empty(world * mine.numel(), dtype=rows32.dtype, device=rows32.device)
        dist.all_gather_into_tensor(allc, mine, group=group)
    for r, (a, b) in enumerate(ranges):
        k = (b - a + GROUP - 1) // GROUP * gw
        rows32[a // GROUP * gw: a // GROUP * gw + k] = allc[r * mine.numel(): r * mine.numel() + k]
    return rows32


# ------------------------------------------------------------------ device pipeline
@dataclass
class StepTimes:
    ms_prepare: float = 0.0
    ms_prefilter: float = 0.0
    ms_mdmc: float = 0.0
    ms_compact: float = 0.0


class DeviceSkycube:
    """Runs the five phases on one GPU; with world > 1 it shards K1, K3 and K4 over the process group."""

    def __init__(self, device: int = 0, group=None):
        self.device = torch.device("cuda", device)
        self.ctx = Context(device)
        self.group = group

    @property
    def launches(self) -> int:
        return self.ctx.launches

    def build(self, pts: torch.Tensor, lists: bool = True, membership: bool = True, events: dict | None = None,
              hashcube_w: int = 0, max_level: int = 0, out_membership: torch.Tensor | None = None,
              out_ids: torch.Tensor | None = None):
        """pts: (n, d) float32 CUDA tensor (resident).  Returns dict of tensors:
        n_ext, shard (j_begin, j_end) of this rank's S+ tasks, rows32 (tiled rows; this rank's range is valid),
        ext_ids, membership [n, W] (optional; with world > 1 only this rank's rows and zero slice are written),
        offsets (global), ids (global positions; with world > 1 only this rank's segments are written),
        total_ids, and with hashcube_w > 0 the HashCube (K5, Appendix B.1).
        max_level = d' > 0: partial skycube (Appendix A.2), only |delta| <= d' reported.
        out_membership / out_ids: caller-provided destinations (device or pinned host tensors: the kernels
        write pinned host memory directly, zero-copy); out_ids must hold total_ids entries."""
        assert pts.is_cuda and pts.dtype == torch.float32 and pts.dim() == 2
        pts = pts.contiguous()
        n, d = pts.shape
        world = _world(self.group)
        rank = dist.get_rank(self.group) if world > 1 else 0
        stream = torch.cuda.current_stream(self.device)
        sp = stream.cuda_stream
        rec = (lambda k: events[k].record(stream)) if events is not None else (lambda k: None)
        W = words_per_row(d)
        nsub = 1 << d

        rec("t0")
        if world == 1:
            self.ctx.prepare(pts.data_ptr(), n, d, sp)
        else:
            # K2 sharded by dimension, the codes all-gathered; the uint32 counts / keys travel as int64 (SUM)
            b, e = dim_slice(d, world, rank)
            per = -(-d // world)
            mine = torch.zeros((per, n), dtype=torch.int16, device=self.device)
            R32 = torch.zeros(d, dtype=torch.int32, device=self.device)
            mo32 = torch.zeros(d, dtype=torch.int32, device=self.device)
            self.ctx.prepare_dims(pts.data_ptr(), n, d, b, e, mine.data_ptr(), R32.data_ptr(), mo32.data_ptr(), sp)
            R64 = R32.to(torch.int64) & 0xffffffff
            mo64 = mo32.to(torch.int64) & 0xffffffff
            codes, Rall, moall = exchange_codes(mine, R64, mo64, d, self.group)
            self.ctx.prepare_finish(codes.data_ptr(), Rall.data_ptr(), moall.data_ptr(), sp)
        rec("t1")
        ext8 = torch.zeros(n, dtype=torch.uint8, device=self.device)
        off, step = prefilter_assignment(rank, world)
        self.ctx.prefilter(ext8.data_ptr(), off, step, sp)
        exchange_ext(ext8, self.group)
        m = self.ctx.set_ext(ext8.data_ptr(), sp)
        rec("t2")
        rows32 = torch.empty(rows_buffer_words(m, d), dtype=torch.int32, device=self.device)
        j0, j1 = task_range(m, world, rank)
        self.ctx.set_max_level(max_level)
        if j1 > j0:
            self.ctx.mdmc(rows32.data_ptr(), j0, j1, 0, sp)
        rec("t3")
        out = {"n_ext": m, "rows32": rows32, "shard": (j0, j1)}
        ext_ids = torch.empty(max(m, 1), dtype=torch.int32, device=self.device)
        self.ctx.compact(rows32.data_ptr(), 0, ext_ids.data_ptr(), 0, 0, sp)
        out["ext_ids"] = ext_ids[:m]
        mem = out_membership
        if mem is None and membership:
            mem = torch.empty((n, W), dtype=torch.int32, device=self.device)
        if mem is not None:
            if world == 1:
                if mem.is_cuda:
                    self.ctx.compact(rows32.data_ptr(), mem.data_ptr(), 0, 0, 0, sp)
                else:
                    self.ctx.membership(rows32.data_ptr(), 0, m, 0, n, mem.data_ptr(), sp)
            else:
                lo, hi = id_slice(n, world, rank)
                self.ctx.membership(rows32.data_ptr(), j0, j1, lo, hi, mem.data_ptr(), sp)
        out["membership"] = mem
        if lists:
            totals = torch.empty(nsub, dtype=torch.int64, device=self.device)
            self.ctx.lattice_count(rows32.data_ptr(), j0, j1, totals.data_ptr(), sp)
            all_totals = exchange_totals(totals, self.group)
            offsets = torch.empty(nsub + 1, dtype=torch.int64, device=self.device)
            total = self.ctx.lattice_scatter(rows32.data_ptr(), j0, j1, all_totals.data_ptr(), world, rank,
                                             offsets.data_ptr(), 0, sp)
            ids = out_ids if out_ids is not None else torch.empty(max(total, 1), dtype=torch.int32, device=self.device)
            assert ids.numel() >= total, "out_ids too small"
            self.ctx.lattice_scatter(rows32.data_ptr(), j0, j1, all_totals.data_ptr(), world, rank, 0,
                                     ids.data_ptr(), sp)
            out["offsets"] = offsets
            out["ids"] = ids[:total]
            out["total_ids"] = total
        if hashcube_w:
            gather_rows(rows32, m, d, self.group)
            nw, nk, ni = self.ctx.hashcube(rows32.data_ptr(), hashcube_w, sp)
            hc = {"word_offsets": torch.empty(nw + 1, dtype=torch.int64, device=self.device),
                  "keys": torch.empty(max(nk, 1), dtype=torch.int32, device=self.device),
                  "key_offsets": torch.empty(nk + 1, dtype=torch.int64, device=self.device),
                  "ids": torch.empty(max(ni, 1), dtype=torch.int32, device=self.device)}
            self.ctx.hashcube_copy(hashcube_w, hc["word_offsets"].data_ptr(), hc["keys"].data_ptr(),
                                   hc["key_offsets"].data_ptr(), hc["ids"].data_ptr(), sp)
            hc["keys"] = hc["keys"][:nk]
            hc["ids"] = hc["ids"][:ni]
            out["hashcube"] = hc
        rec("t4")
        return out

    def close(self):
        self.ctx.close()

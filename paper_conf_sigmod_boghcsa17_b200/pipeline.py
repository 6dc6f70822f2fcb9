"""Per-rank device pipeline of the MDMC skycube, one process per GPU (torch.distributed for plumbing).

Sharding (the paper's device-level data parallelism of MDMC, L308-310, L420 "every
task is independent, there is no need for synchronisation"):

  1. prepare (K0 + key-sum sort + K2 codes)      replicated on every rank (deterministic)
  2. K1 prefilter                                 blocks of 512 static-tree positions,
                                                  block b on rank b % world
  3. exchange S+ flags                            all_reduce(MAX) of a uint8 flag vector (NCCL over NVLink)
  4. install S+ (replicated)
  5. K3 MDMC                                      contiguous ranges of 32-point groups of S+ (per-task cost is
                                                  uniform: every task scans all of S+)
  6. exchange rows                                all_gather of the rank's row chunk (NCCL over NVLink)
  7. K4 compaction                                every rank (identical bytes on every rank)

The collective helpers below are plain torch.distributed calls so that the same code runs on NCCL
(GPU) and gloo (CPU tests).  Only the kernels are native; nothing here computes skycube values.
"""
from __future__ import annotations

import math
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


def groups_per_rank(m: int, world: int) -> int:
    ngroups = math.ceil(m / GROUP) if m > 0 else 0
    return math.ceil(ngroups / world) if ngroups else 0


def task_range(m: int, world: int, rank: int):
    """[j_begin, j_end) of the S+ tasks of a rank (multiples of 32 except the global end)."""
    gpr = groups_per_rank(m, world)
    j0 = min(m, rank * gpr * GROUP)
    j1 = min(m, (rank + 1) * gpr * GROUP)
    return j0, j1


def rows_buffer_words(m: int, d: int, world: int) -> int:
    return max(1, groups_per_rank(m, world) * world) * GROUP * words_per_row(d)


def chunk_words(m: int, d: int, world: int) -> int:
    return groups_per_rank(m, world) * GROUP * words_per_row(d)


# ------------------------------------------------------------------ collectives (NCCL or gloo)
def _staged(t: torch.Tensor, group) -> bool:
    """gloo does not run every collective on CUDA tensors: stage through host memory there (used by the
    single-GPU multi-rank tests; NCCL never stages)."""
    return t.is_cuda and dist.get_backend(group) == "gloo"


def exchange_ext(ext8: torch.Tensor, group=None):
    """Combine per-rank S+ flags: every position was written by exactly one rank, others are 0."""
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        if _staged(ext8, group):
            h = ext8.cpu()
            dist.all_reduce(h, op=dist.ReduceOp.MAX, group=group)
            ext8.copy_(h)
        else:
            dist.all_reduce(ext8, op=dist.ReduceOp.MAX, group=group)
    return ext8


def exchange_rows(rows32: torch.Tensor, m: int, d: int, group=None):
    """All-gather the rank-owned chunks of the tiled row buffer (equal chunk sizes by construction)."""
    if not (dist.is_initialized() and dist.get_world_size(group) > 1):
        return rows32
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    cw = chunk_words(m, d, world)
    if cw == 0:
        return rows32
    mine = rows32[rank * cw:(rank + 1) * cw].clone()
    if _staged(rows32, group):
        h = torch.empty(world * cw, dtype=rows32.dtype)
        dist.all_gather_into_tensor(h, mine.cpu(), group=group)
        rows32[:world * cw].copy_(h)
    else:
        dist.all_gather_into_tensor(rows32[:world * cw], mine, group=group)
    return rows32


# ------------------------------------------------------------------ device pipeline
@dataclass
class StepTimes:
    ms_prepare: float = 0.0
    ms_prefilter: float = 0.0
    ms_mdmc: float = 0.0
    ms_compact: float = 0.0


class DeviceSkycube:
    """Runs the five phases on one GPU; with world > 1 it shards K1 and K3 over the process group."""

    def __init__(self, device: int = 0, group=None):
        self.device = torch.device("cuda", device)
        self.ctx = Context(device)
        self.group = group

    @property
    def launches(self) -> int:
        return self.ctx.launches

    def build(self, pts: torch.Tensor, lists: bool = True, membership: bool = True, events: dict | None = None,
              hashcube_w: int = 0, max_level: int = 0):
        """pts: (n, d) float32 CUDA tensor (resident).  Returns dict of device tensors:
        n_ext, rows32 (tiled rows of S+), ext_ids, membership [n, W] (optional), offsets, ids, and with
        hashcube_w > 0 the HashCube (K5, Appendix B.1) as hashcube = {word_offsets, keys, key_offsets, ids}.
        max_level = d' > 0: partial skycube (Appendix A.2), only |delta| <= d' reported."""
        assert pts.is_cuda and pts.dtype == torch.float32 and pts.dim() == 2
        pts = pts.contiguous()
        n, d = pts.shape
        world = dist.get_world_size(self.group) if dist.is_initialized() else 1
        rank = dist.get_rank(self.group) if dist.is_initialized() else 0
        stream = torch.cuda.current_stream(self.device)
        sp = stream.cuda_stream
        rec = (lambda k: events[k].record(stream)) if events is not None else (lambda k: None)
        W = words_per_row(d)

        rec("t0")
        self.ctx.prepare(pts.data_ptr(), n, d, sp)
        rec("t1")
        ext8 = torch.zeros(n, dtype=torch.uint8, device=self.device)
        off, step = prefilter_assignment(rank, world)
        self.ctx.prefilter(ext8.data_ptr(), off, step, sp)
        exchange_ext(ext8, self.group)
        m = self.ctx.set_ext(ext8.data_ptr(), sp)
        rec("t2")
        rows32 = torch.empty(rows_buffer_words(m, d, world), dtype=torch.int32, device=self.device)
        j0, j1 = task_range(m, world, rank)
        self.ctx.set_max_level(max_level)
        if j1 > j0:
            self.ctx.mdmc(rows32.data_ptr(), j0, j1, 0, sp)
        rec("t3")
        exchange_rows(rows32, m, d, self.group)
        out = {"n_ext": m, "rows32": rows32}
        ext_ids = torch.empty(max(m, 1), dtype=torch.int32, device=self.device)
        mem = torch.empty((n, W), dtype=torch.int32, device=self.device) if membership else None
        self.ctx.compact(rows32.data_ptr(), mem.data_ptr() if mem is not None else 0, ext_ids.data_ptr(), 0, 0, sp)
        out["ext_ids"] = ext_ids[:m]
        out["membership"] = mem
        if lists:
            offsets = torch.empty((1 << d) + 1, dtype=torch.int64, device=self.device)
            total = self.ctx.compact(rows32.data_ptr(), 0, 0, offsets.data_ptr(), 0, sp)
            ids = torch.empty(max(total, 1), dtype=torch.int32, device=self.device)
            self.ctx.compact(rows32.data_ptr(), 0, 0, offsets.data_ptr(), ids.data_ptr(), sp)
            out["offsets"] = offsets
            out["ids"] = ids[:total]
            out["total_ids"] = total
        if hashcube_w:
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

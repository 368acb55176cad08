"""Genome sharding for multi-GPU runs (host logic).

Sites are independent, so the genome is split into contiguous shards, one per
rank.  Rules:

* calibration ownership — a read counts on exactly one rank, the one whose shard holds its
  start, so halo copies are never double-counted when the counts are all-reduced;
* calling halo — a rank calls sites [s0, s1) with every read that can touch them:
  pos in [s0 - L + 1, s1); its reference slice must cover [s0 - L + 1, s1 + L - 1);
* balance — shard boundaries split the cumulative count of aligned bases (read starts x
  length), not the site count, because N gaps and depth vary.
"""
from __future__ import annotations

import numpy as np


def plan_equal(n_sites: int, origin: int, world: int) -> list[tuple[int, int]]:
    """Contiguous shards of (nearly) equal site count."""
    b = [origin + (n_sites * r) // world for r in range(world + 1)]
    return [(b[r], b[r + 1]) for r in range(world)]


def plan_by_bases(pos: np.ndarray, length: np.ndarray, n_sites: int, origin: int,
                  world: int) -> list[tuple[int, int]]:
    """Contiguous shards holding ~equal numbers of aligned bases (by read start)."""
    pos = np.asarray(pos, np.int64)
    if len(pos) == 0 or world == 1:
        return plan_equal(n_sites, origin, world)
    cum = np.cumsum(np.asarray(length, np.int64))
    total = int(cum[-1])
    cuts = [origin]
    for r in range(1, world):
        i = int(np.searchsorted(cum, total * r // world, "left"))
        cuts.append(max(cuts[-1], min(int(pos[min(i, len(pos) - 1)]), origin + n_sites)))
    cuts.append(origin + n_sites)
    return [(cuts[r], cuts[r + 1]) for r in range(world)]


def owned_reads(pos: np.ndarray, s0: int, s1: int) -> tuple[int, int]:
    """Index range of reads whose start lies in [s0, s1) (calibration ownership)."""
    pos = np.asarray(pos)
    return (int(np.searchsorted(pos, np.uint64(s0), "left")),
            int(np.searchsorted(pos, np.uint64(s1), "left")))


def call_reads(pos: np.ndarray, s0: int, s1: int, max_read_len: int) -> tuple[int, int]:
    """Index range of reads that can touch sites [s0, s1): pos in [s0 - L + 1, s1)."""
    pos = np.asarray(pos)
    lo = max(s0 - max_read_len + 1, 0)
    return (int(np.searchsorted(pos, np.uint64(lo), "left")),
            int(np.searchsorted(pos, np.uint64(s1), "left")))


def reference_span(s0: int, s1: int, max_read_len: int, origin: int,
                   n_sites: int) -> tuple[int, int]:
    """Reference coordinates a rank must hold to call [s0, s1) (reads extend L-1 each way)."""
    return (max(origin, s0 - max_read_len + 1), min(origin + n_sites, s1 + max_read_len - 1))


def take_reads(w: dict, ra: int, rb: int) -> dict:
    """Reads [ra, rb) of a workload dict as a standalone read set (offsets rebased to 0)."""
    o0, o1 = int(w["off"][ra]), int(w["off"][rb])
    out = dict(w)
    out.update(pos=w["pos"][ra:rb], len=w["len"][ra:rb], strand=w["strand"][ra:rb],
               hits=w["hits"][ra:rb], off=(np.asarray(w["off"][ra:rb + 1]) - np.uint64(o0)),
               bases=w["bases"][o0:o1], quals=w["quals"][o0:o1])
    return out


def output_offsets(sizes) -> list[int]:
    """Exclusive prefix sum of per-rank output sizes: where each rank's output starts in the
    whole-genome output (records, or words of its compressed stream)."""
    out, acc = [], 0
    for s in sizes:
        out.append(acc)
        acc += int(s)
    return out


def gather_output_offsets(dist, n_local: int, device=None) -> tuple[list[int], int]:
    """SURVEY.md §8(e) collective 2: all-gather every rank's output size (one uint64 each) and
    return (per-rank start offsets, total).  `dist` is torch.distributed with an initialised
    group; `device` is where the one-element tensors live (cuda for NCCL, cpu for gloo)."""
    import torch
    ws = dist.get_world_size()
    mine = torch.tensor([int(n_local)], dtype=torch.int64, device=device)
    allv = torch.empty(ws, dtype=torch.int64, device=device)
    dist.all_gather_into_tensor(allv, mine)
    sizes = [int(x) for x in allv.cpu().tolist()]
    return output_offsets(sizes), sum(sizes)

"""Multi-GPU plumbing (torch.distributed): region sharding and the result gather.

Pairs are independent (PAPER.md's tasks are "pairs of sequences",
L22@4659), so a rank generates and computes its own regions -- no input is
communicated, each rank draws its shard from (config seed, region id) -- and the
path's one exchange step is a single ``all_gather_into_tensor`` of the float64
log10 results, each rank's slot carrying its global pair-id range, after which
rank 0 scatters every result to its global pair index.

Two splits (``shard``):
  * strong (the SURVEY §8e contract for C5): the config's FIXED region set is cut
    into contiguous, whole-region ranges whose cell counts (sum of m*N) are
    balanced over a prefix sum (``split_regions``); the job's output is the same
    2^26 results whatever the GPU count, bitwise (every pair's arithmetic is
    independent of its batch, R14);
  * weak: every rank runs its own ``regions_per_rank`` regions (regions
    rank*k .. rank*k + k - 1).
bench.py and the world-size 2 / 4 gloo tests (tests/test_parallel_cpu.py) run
exactly these functions.
"""
from __future__ import annotations

from typing import Tuple

import numpy as np


def rank_regions(rank: int, world: int, regions_per_rank: int) -> Tuple[int, int]:
    """[start, stop) region ids of ``rank`` (weak scaling: a fixed count per rank)."""
    if not (0 <= rank < world) or regions_per_rank < 1:
        raise ValueError("bad rank/world/regions")
    return rank * regions_per_rank, (rank + 1) * regions_per_rank


def split_regions(n_regions: int, world: int, cells_per_region=None):
    """Strong-scaling split: contiguous region ranges whose cell counts are within one
    region of total/world (greedy over the prefix sum). Returns ``world + 1`` bounds."""
    if cells_per_region is None:
        cells_per_region = np.ones(n_regions)
    c = np.concatenate([[0], np.cumsum(np.asarray(cells_per_region, dtype=np.float64))])
    targets = c[-1] * np.arange(world + 1) / world
    bounds = np.searchsorted(c, targets, side="left")
    # round each cut to the nearer region boundary
    for i in range(1, world):
        b = bounds[i]
        if 0 < b <= n_regions and abs(c[b - 1] - targets[i]) < abs(c[b] - targets[i]):
            bounds[i] = b - 1
    bounds[0], bounds[-1] = 0, n_regions
    return np.maximum.accumulate(bounds).astype(np.int64)


def shard(workload: str, rank: int, world: int, scaling: str, n_regions: int):
    """The regions of ``rank``: returns (r0, r1, pair_start, total_pairs, total_cells, cells).

    strong: ``n_regions`` is the job's fixed region set, split by cells;
    weak: ``n_regions`` regions per rank. pair_start = global index of the rank's first
    pair (pairs are numbered region by region, R x H per region, read-major)."""
    from . import synth

    cfg = synth.CONFIGS[workload]
    if scaling == "strong":
        total = int(n_regions)
        shapes = synth.region_shapes(cfg["spec"], cfg["seed"], 0, total)
        bounds = split_regions(total, world, shapes[:, 4])
        r0, r1 = int(bounds[rank]), int(bounds[rank + 1])
    elif scaling == "weak":
        total = int(n_regions) * world
        shapes = synth.region_shapes(cfg["spec"], cfg["seed"], 0, total)
        r0, r1 = rank_regions(rank, world, int(n_regions))
    else:
        raise ValueError(f"scaling must be 'strong' or 'weak', got {scaling!r}")
    pairs = shapes[:, 0] * shapes[:, 1]
    pair_start = int(pairs[:r0].sum())
    return r0, r1, pair_start, int(pairs.sum()), int(shapes[:, 4].sum()), int(shapes[r0:r1, 4].sum())


def pack_slot(results, pair_start: int, n_slot: int):
    """One rank's gather slot: [pair_start, count, results..., NaN padding] (float64, n_slot + 2
    elements; pair ids < 2^53 are exact in float64)."""
    import torch

    n = int(results.numel())
    if n > n_slot:
        raise ValueError("slot smaller than the rank's results")
    slot = torch.full((n_slot + 2,), float("nan"), dtype=torch.float64, device=results.device)
    slot[0] = float(pair_start)
    slot[1] = float(n)
    slot[2:2 + n] = results
    return slot


def gather_slots(slot, world: int, group=None):
    """The path's one collective: all-gather the equally sized slots into (world, n_slot + 2)."""
    import torch
    import torch.distributed as dist

    out = torch.empty(world * slot.numel(), dtype=slot.dtype, device=slot.device)
    dist.all_gather_into_tensor(out, slot, group=group)
    return out.view(world, slot.numel())


def unpack_global(gathered, total_pairs: int) -> np.ndarray:
    """Rank 0: scatter every rank's results to their global pair ids. Checks that the ranks'
    pair ranges tile [0, total_pairs) exactly once."""
    g = np.asarray(gathered, dtype=np.float64)
    out = np.full(int(total_pairs), np.nan)
    seen = np.zeros(int(total_pairs), dtype=np.int8)
    for row in g:
        s, n = int(row[0]), int(row[1])
        if s < 0 or n < 0 or s + n > total_pairs:
            raise ValueError(f"slot range [{s}, {s + n}) outside [0, {total_pairs})")
        out[s:s + n] = row[2:2 + n]
        seen[s:s + n] += 1
    if not np.all(seen == 1):
        raise ValueError("the ranks' pair ranges do not tile the job exactly once")
    return out

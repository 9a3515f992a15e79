"""Multi-GPU plumbing (torch.distributed): region sharding and the result gather.

Pairs are independent, so a rank generates and computes its own
regions -- no input is communicated -- and the only exchange is one
all-gather of the float64 log10 results (plus their global pair ids) at the end.
Weak scaling: every rank gets the same number of regions.
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
    bounds[0], bounds[-1] = 0, n_regions
    return np.maximum.accumulate(bounds).astype(np.int64)


def gather_results(local, world: int, group=None):
    """All-gather equally sized per-rank result tensors into one (world * n) tensor.
    Ranks with fewer pairs must pad ``local`` to the common size (see ``pad_to``)."""
    import torch
    import torch.distributed as dist

    out = torch.empty(world * local.numel(), dtype=local.dtype, device=local.device)
    dist.all_gather_into_tensor(out, local, group=group)
    return out


def pad_to(x, n: int, value=float("nan")):
    import torch

    if x.numel() == n:
        return x
    out = torch.full((n,), value, dtype=x.dtype, device=x.device)
    out[: x.numel()] = x
    return out


def unpad(gathered, counts):
    """Concatenate the valid prefix of each rank's padded slot (global pair order when
    ranks own consecutive region ranges)."""
    gathered = np.asarray(gathered)
    n = gathered.size // len(counts)
    return np.concatenate([gathered[r * n: r * n + counts[r]] for r in range(len(counts))])

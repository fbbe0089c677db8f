"""Multi-GPU sharding of the kernel axis + NCCL all-gather of the selected-clock table.

Kernels are independent units (one prediction dataset per kernel), so the
kernel axis shards with no exchange on the data path; the only collective assembles the int32
choice table on every rank (BASELINE.json north_star: "an NCCL all-gather over NVLink only to
assemble the selected-frequency table").  One process per GPU, torch.distributed for the
process group.  Models, clock table and targets are replicated (each rank builds them from the
same seeds), predictions stay sharded and are never gathered.

Strong scaling: rank r owns rows [r*per, min(n, (r+1)*per)), per = ceil(n / P); the last shard
is padded to `per` rows (NCCL all-gather needs equal counts, pad rows hold -1) and the padding is
trimmed after the gather.  Weak scaling: every rank owns `per` rows of its own.
"""
from __future__ import annotations

from typing import Callable, Optional, Tuple

import numpy as np


def shard_rows(n_total: int, rank: int, world: int) -> Tuple[int, int, int]:
    """(row0, n_rows, per): rank's contiguous share of n_total rows and the padded shard size."""
    if world < 1 or not (0 <= rank < world) or n_total < 0:
        raise ValueError("bad shard arguments")
    per = (n_total + world - 1) // world
    row0 = min(rank * per, n_total)
    n = max(0, min(n_total, row0 + per) - row0)
    return row0, n, per


class ShardedSweep:
    """Per-rank state for repeated sharded sweeps: a padded local choice buffer and the gathered
    table.  `compute(features_local, out_local)` writes the rank's choices (the CUDA path by
    default; tests inject a CPU stand-in with the gloo backend)."""

    def __init__(self, n_total: int, n_targets: int, rank: int, world: int, device, group=None,
                 compute: Optional[Callable] = None, weak: bool = False):
        import torch
        self.rank, self.world, self.group = rank, world, group
        if weak:
            self.per = n_total
            self.row0, self.n_local = rank * n_total, n_total
            self.n_total = n_total * world
        else:
            self.row0, self.n_local, self.per = shard_rows(n_total, rank, world)
            self.n_total = n_total
        self.n_t = n_targets
        self.local = torch.full((max(self.per, 1), n_targets), -1, dtype=torch.int32, device=device)
        self.table = torch.empty((max(self.per, 1) * world, n_targets), dtype=torch.int32, device=device)
        self.compute = compute

    def run(self, features_local):
        """Sweep the local rows, then all-gather; returns the trimmed [n_total, n_t] table."""
        import torch.distributed as dist
        if self.n_local:
            self.compute(features_local, self.local[:self.n_local])
        if self.world > 1:
            dist.all_gather_into_tensor(self.table, self.local, group=self.group)
        else:
            self.table[:self.per].copy_(self.local[:self.per])
        return self.gathered()

    def gathered(self):
        # rank r's rows are table[r*per : r*per + n_r]; only the tail shards are short (padding
        # at their ends), so the first n_total rows of the gathered table are exactly the data
        return self.table[:self.n_total]


def cuda_compute(speedup, energy, clocks, default_idx, targets):
    """The CUDA path as a ShardedSweep compute function (C ABI synergy_sweep)."""
    from . import synergy as syn

    def fn(features_local, out_local):
        syn.sweep(speedup, energy, features_local, clocks, default_idx, targets, out=out_local)
    return fn


def rank_rows(features_all: np.ndarray, rank: int, world: int) -> np.ndarray:
    row0, n, _ = shard_rows(features_all.shape[0], rank, world)
    return np.ascontiguousarray(features_all[row0:row0 + n])

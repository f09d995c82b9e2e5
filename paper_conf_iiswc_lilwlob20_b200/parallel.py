"""Row-partitioned multi-GPU MTTKRP (the paper lists multi-GPU as future
work).  One process per GPU, ``torch.distributed`` (NCCL over NVLink/NVSwitch) for
the only exchange step: the all-gather of the owned output rows that the next CP-ALS step
needs.

Per target mode n:
  1. nnz-balanced contiguous output-row ranges (``pasta_row_partition``, host C code);
  2. every rank keeps the mode-n sorted shard of its rows (``pasta_coo_shard``) and the
     replicated, read-only factors; MTTKRP on the shard writes only rows [lo, hi) of the
     full-size output (no cross-GPU atomics: rows are exclusively owned);
  3. ``gather_rows``: rank p broadcasts its contiguous row block out[lo_p:hi_p] into every
     replica (an uneven all-gather done in place, no packing copies).
"""
from __future__ import annotations

from typing import List, Sequence

import numpy as np


def gather_rows(out, bounds: Sequence[int], group=None, async_op: bool = False):
    """In-place all-gather(v) of contiguous row blocks: after the call every rank holds
    out[bounds[p]:bounds[p+1]] of every rank p.  Works with NCCL (CUDA tensors) and gloo
    (CPU tensors).  Returns the list of work handles when async_op."""
    import torch.distributed as dist
    works = []
    for p in range(len(bounds) - 1):
        lo, hi = int(bounds[p]), int(bounds[p + 1])
        if hi <= lo:
            continue
        w = dist.broadcast(out[lo:hi], src=p, group=group, async_op=async_op)
        if async_op:
            works.append(w)
    return works


def partition_bounds(counts_per_mode: Sequence[np.ndarray], world: int) -> List[np.ndarray]:
    """nnz-balanced row bounds for every mode (host logic of libpasta, needs no GPU)."""
    from . import pasta_row_partition
    return [pasta_row_partition(np.asarray(c, dtype=np.uint64), world) for c in counts_per_mode]


class RowPartitionedMTTKRP:
    """Holds this rank's per-mode shards of a COO tensor and runs all-mode MTTKRP steps."""

    def __init__(self, x, rank: int, world: int, R: int, device):
        import torch

        from . import pasta_coo_partition, pasta_coo_shard
        self.rank, self.world, self.R = rank, world, R
        self.order, self.dims, self.nnz = x.order, x.dims, x.nnz
        self.bounds = [pasta_coo_partition(x, n, world) for n in range(x.order)]
        self.shards = []
        for n in range(x.order):
            lo, hi = int(self.bounds[n][rank]), int(self.bounds[n][rank + 1])
            self.shards.append(pasta_coo_shard(x, n, lo, hi))
        self.out = [torch.empty((d, R), dtype=torch.float32, device=device) for d in self.dims]

    def shard_nnz(self) -> List[int]:
        return [s.nnz for s in self.shards]

    def step(self, factors, gather: bool = True, stream=None):
        """MTTKRP of every mode on this rank's shards (+ the all-gather of each output
        when world > 1).  The gather of mode n overlaps the compute of mode n + 1."""
        from . import pasta_mttkrp_coo
        works = []
        for n in range(self.order):
            pasta_mttkrp_coo(self.shards[n], n, factors, out=self.out[n], stream=stream)
            if gather and self.world > 1:
                works += gather_rows(self.out[n], self.bounds[n], async_op=True)
        for w in works:
            w.wait()
        return self.out

"""Row-partitioned multi-GPU MTTKRP (the paper lists multi-GPU as future
work).  One process per GPU, ``torch.distributed`` (NCCL over NVLink/NVSwitch) for
the only exchange step: the all-gather of the owned output rows that the next CP-ALS step
needs.

Per target mode n:
  1. nnz-balanced contiguous output-row ranges (``pasta_row_partition``, host C code);
  2. every rank keeps the mode-n sorted shard of its rows (``pasta_coo_shard``) and the
     replicated, read-only factors; MTTKRP on the shard writes only rows [lo, hi) of the
     full-size output (no cross-GPU atomics: rows are exclusively owned);
  3. ``gather_rows``: one padded all-gather per mode of the owned row blocks (NCCL
     all_gather_into_tensor), then each peer block is copied into place.
"""
from __future__ import annotations

from typing import List, Sequence

import numpy as np


_GATHER_BUFS = {}


class _RowGather:
    """One padded all-gather of the owned row blocks: rank p's rows [bounds[p], bounds[p+1])
    travel in slot p of a [P, max_rows, R] buffer (all_gather_into_tensor, a single NCCL
    collective -- NVLS-capable on NVSwitch -- instead of P broadcasts); wait() copies the
    peers' slots into place."""

    def __init__(self, out, bounds, group, async_op):
        import torch.distributed as dist
        self.out, self.bounds = out, [int(b) for b in bounds]
        P = len(self.bounds) - 1
        self.rank = dist.get_rank(group)
        rows = [self.bounds[p + 1] - self.bounds[p] for p in range(P)]
        m = max(max(rows), 1)
        key = (P, m, tuple(out.shape[1:]), out.dtype, str(out.device))
        buf = _GATHER_BUFS.get(key)
        if buf is None:
            buf = out.new_empty((P, m) + tuple(out.shape[1:]))
            _GATHER_BUFS.clear()  # one cached buffer: the shapes of one workload
            _GATHER_BUFS[key] = buf
        self.buf, self.rows = buf, rows
        lo, hi = self.bounds[self.rank], self.bounds[self.rank + 1]
        send = buf[self.rank]
        if hi > lo:
            send[: hi - lo].copy_(out[lo:hi])
        # in place: the input is this rank's slot of the output buffer
        self.work = dist.all_gather_into_tensor(buf.view(-1), send.reshape(-1), group=group,
                                                async_op=async_op)
        if not async_op:
            self._scatter()

    def _scatter(self):
        for p, r in enumerate(self.rows):
            if p != self.rank and r > 0:
                self.out[self.bounds[p]:self.bounds[p + 1]].copy_(self.buf[p, :r])

    def wait(self):
        if self.work is not None:
            self.work.wait()
            self.work = None
            self._scatter()


def gather_rows(out, bounds: Sequence[int], group=None, async_op: bool = False, method: str = "allgather"):
    """All-gather(v) of contiguous row blocks: after the call every rank holds
    out[bounds[p]:bounds[p+1]] of every rank p.  Works with NCCL (CUDA tensors) and gloo (CPU
    tensors).  method "allgather": one padded all_gather_into_tensor (default); "broadcast":
    P in-place broadcasts, no staging buffer.  Returns the list of work handles when async_op."""
    import torch.distributed as dist
    if method == "allgather":
        g = _RowGather(out, bounds, group, async_op)
        return [g] if async_op else []
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
    """Holds this rank's per-mode shards of a COO tensor and runs all-mode MTTKRP steps.
    fmt="hicoo": the shards are HiCOO (pasta_hicoo_shard of the tensor's HiCOO form with
    block_bits, or of `hicoo` when given) and the step runs the HiCOO MTTKRP.  release=True
    frees each mode's full sorted copy of `x` once its shard is cut."""

    def __init__(self, x, rank: int, world: int, R: int, device, fmt: str = "coo", block_bits: int = 7,
                 hicoo=None, release: bool = False):
        import torch

        from . import (pasta_coo_partition, pasta_coo_release_mode, pasta_coo_shard, pasta_coo_to_hicoo,
                       pasta_hicoo_shard)
        self.rank, self.world, self.R, self.fmt = rank, world, R, fmt
        self.order, self.dims, self.nnz = x.order, x.dims, x.nnz
        self.bounds = [pasta_coo_partition(x, n, world) for n in range(x.order)]
        self.shards = []
        h = None
        if fmt == "hicoo":
            h = hicoo if hicoo is not None else pasta_coo_to_hicoo(x, block_bits)
        for n in range(x.order):
            lo, hi = int(self.bounds[n][rank]), int(self.bounds[n][rank + 1])
            self.shards.append(pasta_hicoo_shard(h, n, lo, hi) if h is not None else pasta_coo_shard(x, n, lo, hi))
            if release:  # keep one full sorted copy alive at a time (bounded peak memory)
                pasta_coo_release_mode(x, n)
        del h
        self.out = [torch.empty((d, R), dtype=torch.float32, device=device) for d in self.dims]

    def shard_nnz(self) -> List[int]:
        return [s.nnz for s in self.shards]

    def step_fused(self, factors, replicas, stream=None):
        """MTTKRP of every mode with the all-gather fused into the kernel (COO shards):
        ``replicas`` is a :class:`PeerReplicas` of the output shapes (dims, R); each rank's
        kernel writes its owned rows into every rank's replica (pasta_mttkrp_coo_bcast, P2P
        stores / atomics over NVLink).  A one-element all-reduce after the launches orders the
        peers' reads; the caller orders the previous step's reads before it the same way."""
        import torch

        from . import pasta_mttkrp_coo_bcast
        for n in range(self.order):
            pasta_mttkrp_coo_bcast(self.shards[n], n, factors, replicas.tensors[n], replicas.dsts[n][1:],
                                   stream=stream)
        _all_reduce(torch.zeros(1, dtype=torch.float32, device=factors[0].device))
        return replicas.tensors

    def step(self, factors, gather: bool = True, stream=None):
        """MTTKRP of every mode on this rank's shards (+ the all-gather of each output
        when world > 1).  The gather of mode n overlaps the compute of mode n + 1."""
        from . import pasta_mttkrp_coo, pasta_mttkrp_hicoo
        fn = pasta_mttkrp_hicoo if self.fmt == "hicoo" else pasta_mttkrp_coo
        works = []
        for n in range(self.order):
            fn(self.shards[n], n, factors, out=self.out[n], stream=stream)
            if gather and self.world > 1:
                works += gather_rows(self.out[n], self.bounds[n], async_op=True)
        for w in works:
            w.wait()
        return self.out


def gather_rows_p2p(replicas, k: int, bounds: Sequence[int], rank: int, stream=None) -> None:
    """All-gather of this rank's owned rows [bounds[rank], bounds[rank+1]) of replica k by
    peer stores (pasta_bcast_f32 into every rank's replica).  The caller orders the peers'
    reads after it with a collective."""
    from . import pasta_bcast_f32
    lo, hi = int(bounds[rank]), int(bounds[rank + 1])
    if hi <= lo or len(replicas.dsts[k]) < 2:
        return
    t = replicas.tensors[k]
    R = int(t.shape[1])
    off = lo * R * 4
    pasta_bcast_f32(t[lo:hi], [p + off for p in replicas.dsts[k][1:]], stream=stream)


class PeerReplicas:
    """Replicated factor matrices in IPC-exportable device memory, with every peer's replicas
    mapped into this process (CUDA IPC over NVLink / NVSwitch).  ``tensors[k]`` is this rank's
    [I_k, R] replica; ``dsts[k]`` the device addresses of all ranks' replicas (own first),
    the destination list of :func:`pasta_rows_times_bcast`.  Handles are exchanged once over
    the process group (``all_gather_object``)."""

    def __init__(self, dims, R: int, group=None):
        import torch.distributed as dist

        from . import pasta_dev_alloc, pasta_ipc_get_handle, pasta_ipc_open
        self.own, self.tensors, self.peers = [], [], []
        world = dist.get_world_size(group) if dist.is_initialized() else 1
        rank = dist.get_rank(group) if dist.is_initialized() else 0
        for d in dims:
            t, p = pasta_dev_alloc((int(d), R))
            self.tensors.append(t)
            self.own.append(p)
        handles = [pasta_ipc_get_handle(p) for p in self.own]
        allh = [None] * world
        if world > 1:
            dist.all_gather_object(allh, handles, group=group)
        else:
            allh = [handles]
        self.dsts = []
        for k in range(len(dims)):
            lst = [self.own[k]]
            for q in range(world):
                if q == rank:
                    continue
                ptr = pasta_ipc_open(allh[q][k])
                self.peers.append(ptr)
                lst.append(ptr)
            self.dsts.append(lst)

    def close(self):
        from . import pasta_dev_free, pasta_ipc_close
        for p in self.peers:
            pasta_ipc_close(p)
        self.tensors = []
        for p in self.own:
            pasta_dev_free(p)
        self.own, self.peers, self.dsts = [], [], []


def _all_reduce(t):
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized() and dist.get_world_size() > 1:
        dist.all_reduce(t)
    return t


class RowPartitionedCPALS(RowPartitionedMTTKRP):
    """CP-ALS over row-partitioned MTTKRP: per mode n, each rank computes the
    MTTKRP rows it owns and their R x R gram M_p^T M_p; one all-reduce gives M^T M, from which
    every rank derives the same update matrix Wn, the normalised gram G_n and lambda
    (pasta_cpals_prepare); each rank writes its rows U_n = M Wn, and the owned rows of U_n are
    all-gathered -- the step that makes the output all-gather necessary.
    Every arithmetic step runs in libpasta kernels; only R x R matrices cross the process
    group besides the gathered rows.  fused=False runs the unfused solve / normalise / gram
    sequence (two all-reduces per mode)."""

    def run(self, factors, max_iters=20, tol=1e-5, fused=True, replicas=None):
        """replicas: a :class:`PeerReplicas` whose ``tensors`` are ``factors`` -- the factor
        update then stores every rank's rows straight into all replicas (fused P2P
        all-gather, pasta_rows_times_bcast) instead of NCCL broadcasts."""
        import torch

        from . import (pasta_coo_norm2, pasta_cpals_fit, pasta_cpals_prepare, pasta_cpals_solve, pasta_gram,
                       pasta_mttkrp_coo, pasta_normalize_columns, pasta_rows_times,
                       pasta_rows_times_bcast, pasta_weighted_inner)
        N, R = self.order, self.R
        dev = factors[0].device
        grams = [pasta_gram(u) for u in factors]  # factors are replicated: full grams locally
        # ||X||^2: the mode-0 shards partition the nonzeros
        normx2 = _all_reduce(torch.tensor([pasta_coo_norm2(self.shards[0])], dtype=torch.float64,
                                          device=dev)).item()
        lam = torch.ones(R, dtype=torch.float64, device=dev)
        fits = []
        for it in range(max_iters):
            for n in range(N):
                lo, hi = int(self.bounds[n][self.rank]), int(self.bounds[n][self.rank + 1])
                M = pasta_mttkrp_coo(self.shards[n], n, factors, out=self.out[n])
                others = [grams[k] for k in range(N) if k != n]
                if fused:
                    GM = _all_reduce(pasta_gram(M[lo:hi]))
                    Wn, grams[n], lam = pasta_cpals_prepare(GM, others)
                    if replicas is not None:
                        # every rank finished reading U_n (its MTTKRPs precede the all-reduce
                        # above); after the P2P stores, a collective orders the peers' reads
                        pasta_rows_times_bcast(M, lo, hi, Wn, replicas.dsts[n])
                        _all_reduce(torch.zeros(1, dtype=torch.float64, device=dev))
                        continue
                    pasta_rows_times(M[lo:hi], Wn, U=factors[n][lo:hi])
                    if self.world > 1:
                        gather_rows(factors[n], self.bounds[n])
                    continue
                colsq = torch.zeros(R, dtype=torch.float64, device=dev)
                pasta_cpals_solve(M[lo:hi], others, U=factors[n][lo:hi], colsq=colsq)
                _all_reduce(colsq)
                lam = pasta_normalize_columns(factors[n][lo:hi], colsq, lam=lam)
                g = pasta_gram(factors[n][lo:hi])
                grams[n] = _all_reduce(g)
                if self.world > 1:
                    gather_rows(factors[n], self.bounds[n])
            lo, hi = int(self.bounds[N - 1][self.rank]), int(self.bounds[N - 1][self.rank + 1])
            inner = _all_reduce(pasta_weighted_inner(self.out[N - 1][lo:hi],
                                                     factors[N - 1][lo:hi], lam))
            fits.append(pasta_cpals_fit(grams, lam, inner, normx2))  # fit algebra in a kernel
            if it > 0 and abs(fits[-1] - fits[-2]) < tol:
                break
        return lam.cpu().numpy(), fits

"""The N > 1 path on CPU: world_size-2 `gloo` process group standing in for NCCL.

Each rank owns the nnz-balanced row range that libpasta's host partitioner assigns it
(pasta_row_partition), computes only those output rows (here with the oracle, since the
build box has no GPU), and the in-place uneven all-gather (parallel.gather_rows) must
reassemble exactly the full single-process result on every rank.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth_inputs as si


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, result_q, method):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import paper_conf_iiswc_lilwlob20_b200 as pasta
        from paper_conf_iiswc_lilwlob20_b200.parallel import gather_rows, partition_bounds

        dims = (700, 300, 500)
        inds, vals = si.hot_row_coo(dims, 3000, 20000, seed=5, mode=0, hot_row=3)
        R = 8
        U = si.factors(dims, R, seed=2)
        counts = [np.bincount(inds[n], minlength=dims[n]).astype(np.uint64) for n in range(3)]
        bounds = partition_bounds(counts, world)
        ok = True
        for n in range(3):
            lo, hi = int(bounds[n][rank]), int(bounds[n][rank + 1])
            mine = (inds[n] >= lo) & (inds[n] < hi)
            part, _ = oracle.mttkrp(dims, np.ascontiguousarray(inds[:, mine]), vals[mine], n, U)
            out = torch.full((dims[n], R), float("nan"), dtype=torch.float32)
            out[lo:hi] = torch.from_numpy(part[lo:hi].astype(np.float32))
            gather_rows(out, bounds[n], method=method)
            full, _ = oracle.mttkrp(dims, inds, vals, n, U)
            ok &= bool(np.allclose(out.numpy(), full.astype(np.float32), rtol=0, atol=0))
            # the shards are disjoint and cover every nonzero
            tot = torch.tensor([int(mine.sum())])
            dist.all_reduce(tot)
            ok &= int(tot.item()) == vals.shape[0]
        result_q.put((rank, ok))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("method", ["allgather", "broadcast"])
def test_row_partitioned_allgather_world2(method):
    world = 2
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, method)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert all(p.exitcode == 0 for p in procs)
    assert all(ok for _, ok in res), res

"""Worker for tests/test_gpu_multirank.py: 2 ranks (torchrun) sharing cuda:0 over gloo run the
row-partitioned MTTKRP (shards + in-place all-gather) and compare against the oracle."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import oracle  # noqa: E402
import paper_conf_iiswc_lilwlob20_b200 as pasta  # noqa: E402
import synth_inputs as si  # noqa: E402
from paper_conf_iiswc_lilwlob20_b200.parallel import RowPartitionedMTTKRP  # noqa: E402


def main():
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    torch.cuda.set_device(0)
    dist.init_process_group("gloo")
    dims = (4000, 900, 2500)
    inds, vals = si.hot_row_coo(dims, 40_000, 160_000, seed=33, mode=1, hot_row=7)
    U = si.factors(dims, 16, seed=9)
    Ud = [torch.from_numpy(u).cuda() for u in U]
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    ok = True
    for fmt in ("coo", "hicoo"):  # COO shards, and HiCOO shards (pasta_hicoo_shard)
        part = RowPartitionedMTTKRP(x, rank, world, 16, torch.device("cuda", 0), fmt=fmt)
        outs = part.step(Ud, gather=True)
        torch.cuda.synchronize()
        for n in range(3):
            ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
            g = outs[n].cpu().numpy().astype(np.float64)
            ok &= bool(np.all(np.abs(g - ref) <= 1e-4 * ab + 1e-6))
    # fused MTTKRP + all-gather over peer memory (CUDA IPC replicas; two ranks on one GPU here)
    from paper_conf_iiswc_lilwlob20_b200.parallel import PeerReplicas
    part = RowPartitionedMTTKRP(x, rank, world, 16, torch.device("cuda", 0))
    reps = PeerReplicas(dims, 16)
    for t in reps.tensors:
        t.fill_(float("nan"))  # every row must be written by its owner
    torch.cuda.synchronize()
    dist.barrier()
    outs = part.step_fused(Ud, reps)
    torch.cuda.synchronize()
    for n in range(3):
        ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
        g = outs[n].cpu().numpy().astype(np.float64)
        ok &= bool(np.all(np.abs(g - ref) <= 1e-4 * ab + 1e-6))
    dist.barrier()
    reps.close()
    flag = torch.tensor([1 if ok else 0])
    dist.all_reduce(flag, op=dist.ReduceOp.MIN)
    dist.destroy_process_group()
    sys.exit(0 if int(flag.item()) == 1 else 3)


if __name__ == "__main__":
    main()

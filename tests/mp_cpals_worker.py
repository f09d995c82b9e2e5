"""Worker for tests/test_gpu_multirank.py: 2 ranks sharing cuda:0 (gloo) run the
row-partitioned CP-ALS and must match the single-process CP-ALS oracle's fit.
PASTA_TEST_EXCHANGE=p2p: factors live in IPC-exportable replicas and the factor update
stores every rank's rows into both replicas (pasta_rows_times_bcast through CUDA IPC);
=unfused: the solve / normalise / gram sequence with NCCL-style broadcasts."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import paper_conf_iiswc_lilwlob20_b200 as pasta  # noqa: E402
import synth_inputs as si  # noqa: E402
from oracle.cpals import cp_als  # noqa: E402
from paper_conf_iiswc_lilwlob20_b200.parallel import RowPartitionedCPALS  # noqa: E402


def main():
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    torch.cuda.set_device(0)
    dist.init_process_group("gloo")
    dims, R = (300, 200, 250), 8
    inds, vals = si.powerlaw_coo(dims, 30000, seed=12)
    U0 = si.factors(dims, R, seed=13)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    runner = RowPartitionedCPALS(x, rank, world, R, torch.device("cuda", 0))
    mode = os.environ.get("PASTA_TEST_EXCHANGE", "nccl")
    reps = None
    if mode == "p2p":
        from paper_conf_iiswc_lilwlob20_b200.parallel import PeerReplicas
        reps = PeerReplicas(dims, R)
        for k in range(len(dims)):
            reps.tensors[k].copy_(torch.from_numpy(U0[k]))
        torch.cuda.synchronize()
        dist.barrier()
        Ud = reps.tensors
    else:
        Ud = [torch.from_numpy(u.copy()).cuda() for u in U0]
    lam, fits = runner.run(Ud, max_iters=3, tol=0.0, fused=(mode != "unfused"), replicas=reps)
    if reps is not None:
        torch.cuda.synchronize()
        dist.barrier()
        # both replicas hold identical factors after the fused exchange
        local = [t.cpu() for t in reps.tensors]
        allf = [None] * world
        dist.all_gather_object(allf, [t.numpy() for t in local])
        same = all(np.array_equal(allf[0][k], allf[q][k]) for q in range(world) for k in range(len(dims)))
        # the plain P2P all-gather of owned rows: rank-tagged rows land in every replica
        from paper_conf_iiswc_lilwlob20_b200.parallel import gather_rows_p2p
        b = runner.bounds[0]
        lo, hi = int(b[rank]), int(b[rank + 1])
        reps.tensors[0][lo:hi] = float(rank + 1)
        torch.cuda.synchronize()
        dist.barrier()
        gather_rows_p2p(reps, 0, b, rank)
        torch.cuda.synchronize()
        dist.barrier()
        t0 = reps.tensors[0].cpu()
        for q in range(world):
            same = same and bool((t0[int(b[q]):int(b[q + 1])] == float(q + 1)).all())
        dist.barrier()
        reps.close()
        if not same:
            print("replicas differ", flush=True)
            sys.exit(4)
    _, lam_o, fits_o = cp_als(dims, inds, vals, U0, iters=3)
    ok = np.allclose(fits, fits_o, atol=2e-4) and np.allclose(lam, lam_o, rtol=2e-3)
    flag = torch.tensor([1 if ok else 0])
    dist.all_reduce(flag, op=dist.ReduceOp.MIN)
    dist.destroy_process_group()
    sys.exit(0 if int(flag.item()) == 1 else 3)


if __name__ == "__main__":
    main()

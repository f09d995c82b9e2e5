"""The N > 1 path on one GPU: torchrun launches 2 ranks that share cuda:0 over gloo (NCCL
refuses two ranks per GPU).  Checks the row-partitioned runner end to end (shards, kernel
writes of owned rows, in-place all-gather) and bench.py's multi-rank code path (barrier,
max-over-ranks timing, rank-0-only JSON line, reference arm)."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _torchrun(args, env_extra=None, timeout=600):
    env = dict(os.environ, **(env_extra or {}))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_port())] + args
    return subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=timeout)


def test_row_partitioned_two_ranks_gloo():
    r = _torchrun([os.path.join(ROOT, "tests", "mp_rowpart_worker.py")])
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]


def _bench(args, env_extra=None, timeout=1200):
    """bench.py --gpus 2 outside torchrun: bench.py re-launches itself with 2 ranks."""
    env = dict(os.environ, **(env_extra or {}))
    env.pop("WORLD_SIZE", None)
    r = subprocess.run([sys.executable, "bench.py"] + args, cwd=ROOT, env=env, capture_output=True,
                       text=True, timeout=timeout)
    assert r.returncode == 0, r.stderr[-4000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout  # rank 0 only
    return json.loads(lines[0])


def test_bench_two_ranks_shared_gpu_weak():
    d = _bench(["--gpus", "2", "--config", "c4", "--steps", "3", "--warmup", "3", "--no-cpu-baseline"],
               {"PASTA_BENCH_SHARED_GPU": "1"})
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["scaling"] == "weak"
    assert d["config"]["nnz"] == 2 * 54_000_000  # the tensor grows with the GPU count
    ag = d["allgather"]
    assert ag["ms_per_step"] > 0 and ag["bytes_received_per_rank"] > 0 and ag["broadcast"]["ms_per_step"] > 0
    assert ag["p2p"]["ms_per_step"] > 0 and ag["fused"]["ms_per_step"] > 0  # CUDA IPC on one GPU
    assert d["e2e"]["value"] > 0 and d["gpu_launches"] > 0
    assert 0 < d["roofline"]["frac"] < 1.0  # compulsory bytes of this rank's launches
    bal = d["shard_max_over_mean"]  # nnz-balanced row ranges: max / mean nonzeros per rank
    assert len(bal) == 4 and all(1.0 <= b < 1.05 for b in bal), bal
    r2 = _torchrun(["bench.py", "--impl", "reference", "--gpus", "2", "--config", "c1",
                    "--steps", "2", "--warmup", "3", "--ref-block", "2000"])
    assert r2.returncode == 0, r2.stderr[-4000:]
    lines = [l for l in r2.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1 and json.loads(lines[0])["impl"] == "reference"


def test_bench_two_ranks_shared_gpu_strong_c5():
    """BASELINE config 5 (1B nonzeros, R = 32) split over 2 ranks sharing cuda:0: strong
    scaling, each rank holding only its shards, T_1 timed by rank 0 before sharding."""
    d = _bench(["--gpus", "2", "--config", "c5", "--steps", "3", "--warmup", "3", "--no-cpu-baseline",
                "--e2e-steps", "1"], {"PASTA_BENCH_SHARED_GPU": "1"})
    assert d["n_gpus"] == 2 and d["scaling"] == "strong" and d["config"]["nnz"] == 1_000_000_000
    st = d["strong_scaling"]
    assert st["t1_ms_per_step"] > 0 and st["tp_ms_per_step"] > 0 and st["t1_over_p_tp"] > 0
    assert d["max_shard_nnz"] < 0.55e9  # a rank holds about half of the nonzeros of a mode
    assert all(1.0 <= b < 1.05 for b in d["shard_max_over_mean"])


@pytest.mark.parametrize("exchange", ["nccl", "unfused", "p2p"])
def test_row_partitioned_cpals_two_ranks_gloo(exchange):
    """exchange = p2p: the fused factor update + all-gather over CUDA-IPC peer memory."""
    r = _torchrun([os.path.join(ROOT, "tests", "mp_cpals_worker.py")], {"PASTA_TEST_EXCHANGE": exchange})
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]

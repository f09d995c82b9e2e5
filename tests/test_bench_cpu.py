"""bench.py's host-side paths on CPU: the --gpus N self-launch under torch.distributed.run
(world size 2, 127.0.0.1) with the reference arm, where rank 0 alone prints one JSON line."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_two_ranks_self_launch():
    env = dict(os.environ)
    env.pop("WORLD_SIZE", None)
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--gpus", "2", "--config", "c1",
                        "--steps", "2", "--warmup", "3", "--ref-block", "4000"], cwd=ROOT, env=env,
                       capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["n_gpus"] == 2 and d["config"]["same_config"]
    assert d["cpu_baseline"]["cores"] == 1 and d["config"]["nnz"] == 2 * 10_000
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["value"] > 0

"""bench.py's multi-rank entry point on CPU (-m "not gpu"): `python bench.py --gpus 2` with no
torchrun environment re-launches itself under torch.distributed.run (2 ranks, rendezvous on
127.0.0.1, gloo without a GPU) -- the launch the driver's scaling run uses -- and rank 0
alone prints one JSON line carrying n_gpus = 2 and the max-over-ranks time."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(*args, env=None):
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                          timeout=300, env=dict(os.environ, **(env or {})))


def test_gpus2_spawns_two_ranks():
    r = _run("--gpus", "2", "--dry-run", env={"CUDA_VISIBLE_DEVICES": ""})
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["max_over_ranks"] == 2.0
    assert sorted(s[0] for s in d["shards"]) == [0, 1]
    assert [s[1] for s in sorted(d["shards"])] == [0, 8192]      # weak shards: rank r serves rows r*8192..


def test_world_size_mismatch_is_rejected():
    r = _run("--gpus", "2", "--dry-run", env={"WORLD_SIZE": "1", "RANK": "0"})
    assert r.returncode != 0 and "WORLD_SIZE" in (r.stderr + r.stdout)

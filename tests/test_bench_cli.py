"""bench.py launch contract (host logic, no GPU): `--gpus N` without a torchrun environment
self-launches N ranks and fails loudly when the node has fewer than N devices; a torchrun
environment whose WORLD_SIZE disagrees with --gpus is rejected."""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
torch = pytest.importorskip("torch")


def _bench(args, env_extra):
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    env.update(env_extra)
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], env=env,
                          capture_output=True, text=True, timeout=300)


@pytest.mark.skipif(torch.cuda.is_available() and torch.cuda.device_count() >= 64, reason="needs < 64 GPUs")
def test_too_many_gpus_fails_loudly():
    r = _bench(["--gpus", "64", "--steps", "1", "--warmup", "3"], {})
    assert r.returncode != 0
    assert "needs 64 CUDA devices" in r.stderr


def test_world_size_mismatch_rejected():
    r = _bench(["--gpus", "2", "--steps", "1"], {"WORLD_SIZE": "1", "RANK": "0"})
    assert r.returncode != 0 and "WORLD_SIZE=1" in r.stderr

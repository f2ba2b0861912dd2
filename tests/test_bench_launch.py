"""bench.py launch contract on a host without enough GPUs (CPU only): a
multi-GPU request never silently runs one GPU."""

import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, env_extra):
    env = dict(os.environ, **env_extra)
    for k in ("WORLD_SIZE", "RANK", "LOCAL_RANK"):
        if k not in env_extra:
            env.pop(k, None)
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, env=env,
                          capture_output=True, text=True, timeout=300)


def test_gpus_n_without_devices_fails_loudly():
    import torch
    if torch.cuda.device_count() >= 2:
        pytest.skip("this host has the GPUs: bench.py would launch for real")
    r = _run(["--gpus", "2", "--steps", "1", "--warmup", "3"], {"CUDA_VISIBLE_DEVICES": ""})
    assert r.returncode == 2, r.stderr
    assert "needs 2 CUDA devices" in r.stderr
    assert '"n_gpus"' not in r.stdout


def test_world_size_mismatch_fails_loudly():
    r = _run(["--gpus", "2", "--steps", "1", "--warmup", "3"], {"WORLD_SIZE": "3", "RANK": "0"})
    assert r.returncode == 2
    assert "WORLD_SIZE=3 but --gpus 2" in r.stderr
    r = _run(["--gpus", "1", "--steps", "1", "--warmup", "3"], {"WORLD_SIZE": "2", "RANK": "0"})
    assert r.returncode == 2

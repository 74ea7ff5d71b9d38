"""bench.py's launcher logic without a GPU (`bench.py --gpus N` must never report a
smaller run as N GPUs)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, env_extra=None, timeout=240):
    env = {k: v for k, v in os.environ.items() if k not in ("RANK", "WORLD_SIZE", "LOCAL_RANK", "MASTER_PORT")}
    env.update(env_extra or {})
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True, text=True,
                          timeout=timeout, env=env, cwd=ROOT)


def test_gpus_without_enough_devices_fails_loudly():
    """`--gpus 2` outside torchrun starts 2 rank processes itself; with fewer GPUs visible each
    rank refuses, and the launcher exits non-zero without printing a bench line."""
    torch = pytest.importorskip("torch")
    if torch.cuda.is_available() and torch.cuda.device_count() >= 2:
        pytest.skip("this box has 2 GPUs")
    r = _run(["--gpus", "2", "--steps", "1", "--warmup", "3", "--no-slowdown", "--no-cpu-baseline"])
    assert r.returncode != 0
    assert "GPUs" in r.stderr and '"metric"' not in r.stdout


def test_world_size_must_match_gpus():
    r = _run(["--gpus", "2", "--steps", "1"], {"RANK": "0", "WORLD_SIZE": "1", "LOCAL_RANK": "0"})
    assert r.returncode != 0 and "refusing" in r.stderr


def test_reference_arm_prints_one_line():
    """--impl reference: the CPU oracle on a bounded sample of the default (C3) workload."""
    r = _run(["--impl", "reference", "--steps", "1", "--warmup", "0"])
    assert r.returncode == 0, r.stderr[-2000:]
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["config"]["config"] == "c3" and line["unit"] == "GB/s"
    assert line["cpu_baseline"]["kind"] == "oracle" and line["e2e"]["h2d_bytes_per_step"] == 0

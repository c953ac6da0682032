"""bench.py launcher (VERDICT r1 "Next" 2): `python bench.py --gpus N` outside torchrun
starts the N ranks itself; under torchrun the world size must equal --gpus.
CPU only: the reference arm (oracle) needs no GPU, so the two-rank launch runs here."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


class _A:
    def __init__(self, gpus, backend="nccl"):
        self.gpus, self.backend = gpus, backend


def test_launch_command_shape():
    cmd = bench.launch_command(["--gpus", "4", "--steps", "2"], 4, 29512)
    assert cmd[1:3] == ["-m", "torch.distributed.run"]
    assert "--nproc-per-node=4" in cmd and "--nnodes=1" in cmd
    assert cmd[cmd.index("--master-addr") + 1] == "127.0.0.1"
    assert cmd[cmd.index("--master-port") + 1] == "29512"
    assert cmd[-4:] == ["--gpus", "4", "--steps", "2"] and cmd[-5].endswith("bench.py")


def test_self_launch_noop_for_one_gpu(monkeypatch):
    monkeypatch.delenv("WORLD_SIZE", raising=False)
    assert bench.self_launch(_A(1), ["--gpus", "1"]) is None


def test_self_launch_under_torchrun_checks_world(monkeypatch):
    monkeypatch.setenv("WORLD_SIZE", "2")
    assert bench.self_launch(_A(2), ["--gpus", "2"]) is None
    with pytest.raises(SystemExit):
        bench.self_launch(_A(4), ["--gpus", "4"])


def test_two_ranks_without_torchrun():
    """End to end on CPU: --gpus 2 with no torchrun wrapper runs two ranks; rank 0 prints one JSON line
    reporting n_gpus = 2 (reference arm: the oracle on a tiny sample)."""
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--gpus", "2",
                        "--config", "C1", "--steps", "1", "--warmup", "0", "--cpu-voxels", "2"],
                       capture_output=True, text=True, timeout=600, env=env, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [json.loads(ln) for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    assert lines[0]["n_gpus"] == 2 and lines[0]["impl"] == "reference"

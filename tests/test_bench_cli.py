"""bench.py's launch contract, on CPU: --gpus N > 1 without a torchrun environment re-executes the same
command under torch.distributed.run with N processes on 127.0.0.1 (one rank per GPU); under torchrun
(RANK set) it runs as that rank."""
import json
import os
import subprocess
import sys

from conftest import ROOT

BENCH = os.path.join(ROOT, "bench.py")


def _run(args, env=None):
    e = {k: v for k, v in os.environ.items() if k not in ("RANK", "WORLD_SIZE", "LOCAL_RANK")}
    e.update(env or {})
    out = subprocess.run([sys.executable, BENCH] + args, env=e, capture_output=True, text=True, timeout=120)
    assert out.returncode == 0, out.stderr
    return json.loads(out.stdout.strip().splitlines()[-1])


def test_gpus_n_relaunches_under_torchrun():
    r = _run(["--gpus", "2", "--steps", "3", "--warmup", "3", "--dry-run"])
    cmd = r["launch"]
    assert cmd[1:3] == ["-m", "torch.distributed.run"]
    assert "--nproc-per-node=2" in cmd and "127.0.0.1" in cmd
    assert cmd[cmd.index(BENCH) + 1:] == ["--gpus", "2", "--steps", "3", "--warmup", "3", "--dry-run"]


def test_rank_environment_runs_in_place():
    r = _run(["--gpus", "2", "--dry-run"], env={"RANK": "1", "WORLD_SIZE": "2", "LOCAL_RANK": "1"})
    assert r == {"launch": None, "rank": 1, "world": 2}
    r = _run(["--dry-run"])
    assert r == {"launch": None, "rank": 0, "world": 1}

"""The library's world > 1 path, executed (SURVEY.md §8e; PAPER.md:539 §5.3 scale-up, :791 App. C).

Two processes share the test box's one GPU, so the collective is the caller-supplied allreduce of
vista_sys_cfg (a gloo process group) instead of NCCL, which refuses two ranks on one device.  Every
LR pass and MLP step of both ranks goes through it: vista_plan(world = 2) -> vista_transfer on the
rank's image shard -> vista_train(k) / vista_train_mlp(k).  Compared with world = 1 over the union:

* join pairs and every MM_k row: bit-exact (rows are independent; the union of the ranks' pairs is the
  world-1 pair set);
* LR weights, loss, lambda_hat: within 1e-5 relative.  Not bit-exact: each rank's fp32 in-CTA partial
  sums cover a different row subset than world 1's CTAs do, so the fp64 totals differ
  at fp32 rounding level (~1e-7);
* a rank with NO images (hence no train rows) takes part in every collective with zero partials: the
  totals are then world 1's sums + 0.0, so the weights are bit-identical to world 1 on rank 0's rows
  run through the same (unfused: partials -> reduce -> allreduce -> update) LR kernels, for the LR and
  for the MLP (this is the rank that used to leave the MLP deadlocked);
* world 1's default LR (reduce + update fused into the pass kernels, cooperative grid barriers) agrees
  with that unfused sequence to 1e-12 relative (only the order of the fp64 update sums differs).
"""
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

from conftest import ROOT

pytestmark = pytest.mark.gpu
WORKER = os.path.join(ROOT, "tests", "mr_worker.py")


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _run(out, world, N, n0, mlp, **extra_env):
    env = dict(os.environ, MASTER_ADDR="127.0.0.1", MASTER_PORT=str(_port()), WORLD_SIZE=str(world), **extra_env)
    procs = []
    for r in range(world):
        e = dict(env, RANK=str(r), LOCAL_RANK=str(r))
        procs.append(subprocess.Popen([sys.executable, WORKER, str(out), str(N), str(n0), str(mlp)], env=e,
                                      stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True))
    logs = []
    for p in procs:
        try:
            o, _ = p.communicate(timeout=600)
        except subprocess.TimeoutExpired:
            p.kill()
            o, _ = p.communicate()
        logs.append(o)
    for p, o in zip(procs, logs):
        assert p.returncode == 0, o[-3000:]
    return [dict(np.load(os.path.join(out, f"rank{r}.npz"))) for r in range(world)]


def _rows(res, k):
    """{(str_row, global img_row): MM row bytes} over the ranks' results."""
    d = {}
    for r in res:
        for p, (s, i) in enumerate(zip(r[f"pair_str{k}"], r[f"pair_img{k}"])):
            d[(int(s), int(i))] = r[f"mm{k}"][p].tobytes()
    return d


def _rel(a, b):
    return np.linalg.norm(a - b) / max(np.linalg.norm(b), 1e-300)


@pytest.fixture(scope="module")
def world1(tmp_path_factory):
    out = tmp_path_factory.mktemp("w1")
    return _run(out, 1, 240, 240, 1)[0]


def test_world2_split_matches_world1(tmp_path, world1):
    res = _run(tmp_path, 2, 240, 100, 1)
    for k in range(3):
        # join + concat: the union of the shards' rows is the world-1 result, bit for bit
        assert _rows(res, k) == _rows([world1], k)
        assert sum(int(r[f"n_train{k}"][0]) for r in res) == int(world1[f"n_train{k}"][0])
        # the collective made the model identical on both ranks
        np.testing.assert_array_equal(res[0][f"w{k}"], res[1][f"w{k}"])
        assert _rel(res[0][f"w{k}"], world1[f"w{k}"]) <= 1e-5
        np.testing.assert_allclose(res[0][f"loss{k}"], world1[f"loss{k}"], rtol=1e-6)
        np.testing.assert_allclose(res[0][f"met{k}"][0], world1[f"met{k}"][0], rtol=1e-6)  # lambda_hat
        np.testing.assert_array_equal(res[0][f"met{k}"][1:3], world1[f"met{k}"][1:3])      # n_train, n_test
        assert np.abs(res[0][f"met{k}"][3:] - world1[f"met{k}"][3:]).sum() <= 2            # confusion counts
    for name in ("mlp_W1", "mlp_W2", "mlp_w3"):
        np.testing.assert_array_equal(res[0][name], res[1][name])
        assert _rel(res[0][name], world1[name]) <= 1e-4
    np.testing.assert_allclose(res[0]["mlp_loss"], world1["mlp_loss"], rtol=1e-5)


def test_world2_with_an_empty_rank(tmp_path):
    # rank 1 owns no images: zero train rows, zero pairs; every collective still completes and adds 0.0,
    # so the model equals world 1 on rank 0's images bit for bit (LR and MLP)
    (tmp_path / "ref").mkdir()
    (tmp_path / "fused").mkdir()
    ref = _run(tmp_path / "ref", 1, 150, 150, 1, VISTA_LR_FUSED="0")[0]
    fused = _run(tmp_path / "fused", 1, 150, 150, 1)[0]
    res = _run(tmp_path, 2, 150, 150, 1)
    assert int(res[1]["n_train0"][0]) == 0 and len(res[1]["pair_str0"]) == 0
    for k in range(3):
        np.testing.assert_array_equal(res[0][f"w{k}"], ref[f"w{k}"])
        np.testing.assert_array_equal(res[1][f"w{k}"], ref[f"w{k}"])
        np.testing.assert_array_equal(res[0][f"loss{k}"], ref[f"loss{k}"])
        np.testing.assert_array_equal(res[1][f"met{k}"], ref[f"met{k}"])
    for name in ("mlp_W1", "mlp_W2", "mlp_w3", "mlp_loss", "mlp_met"):
        np.testing.assert_array_equal(res[0][name], ref[name])
        np.testing.assert_array_equal(res[1][name], ref[name])
    for k in range(3):  # fused world-1 LR vs the unfused kernels
        assert _rel(fused[f"w{k}"], ref[f"w{k}"]) <= 1e-12
        np.testing.assert_allclose(fused[f"loss{k}"], ref[f"loss{k}"], rtol=1e-12)
        np.testing.assert_array_equal(fused[f"met{k}"][1:], ref[f"met{k}"][1:])

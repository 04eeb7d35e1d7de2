"""Pins of the MLP oracle (oracle/mlp.py; "3-layer MLP (each hidden layer has 1024
units) for 10 iterations"; reading R30) against things other than itself:
central finite differences, torch autograd in fp64 (library), the W1 = W2 = 0 special case
(scalar recursion of the bias), the descent property, and a world-2 gloo data-parallel run
whose allreduced shard gradients equal the full-batch gradient."""
import os
import socket

import numpy as np
import pytest
import torch

import gen
import oracle
from oracle import mlp

rng = np.random.default_rng(7)


def small_problem(n=9, d=6, h=5):
    X = rng.standard_normal((n, d))
    y = (rng.random(n) < 0.5).astype(np.uint8)
    P = dict(W1=rng.standard_normal((h, d)) * 0.7, b1=rng.standard_normal(h) * 0.3,
             W2=rng.standard_normal((h, h)) * 0.7, b2=rng.standard_normal(h) * 0.3,
             w3=rng.standard_normal(h), b3=0.2)
    return X, y, P


def test_gradient_matches_central_differences():
    X, y, P = small_problem()
    _, g = mlp.loss_and_grad(P, X, y)
    eps = 1e-6
    for k in P:
        if np.isscalar(P[k]):
            Pp, Pm = dict(P), dict(P)
            Pp[k], Pm[k] = P[k] + eps, P[k] - eps
            fd = (mlp.loss_and_grad(Pp, X, y)[0] - mlp.loss_and_grad(Pm, X, y)[0]) / (2 * eps)
            assert abs(fd - g[k]) <= 1e-7 * max(1.0, abs(fd))
            continue
        flat = P[k].reshape(-1)
        for i in range(flat.size):
            Pp = {kk: (v.copy() if not np.isscalar(v) else v) for kk, v in P.items()}
            Pm = {kk: (v.copy() if not np.isscalar(v) else v) for kk, v in P.items()}
            Pp[k].reshape(-1)[i] += eps
            Pm[k].reshape(-1)[i] -= eps
            fd = (mlp.loss_and_grad(Pp, X, y)[0] - mlp.loss_and_grad(Pm, X, y)[0]) / (2 * eps)
            assert abs(fd - g[k].reshape(-1)[i]) <= 1e-7 * max(1.0, abs(fd)), (k, i)


def test_gradient_matches_torch_autograd():
    X, y, P = small_problem(n=40, d=12, h=16)
    loss, g = mlp.loss_and_grad(P, X, y)
    T = {k: torch.tensor(v, dtype=torch.float64, requires_grad=True) for k, v in P.items()}
    Xt = torch.from_numpy(X)
    h1 = torch.relu(Xt @ T["W1"].T + T["b1"])
    h2 = torch.relu(h1 @ T["W2"].T + T["b2"])
    z = h2 @ T["w3"] + T["b3"]
    lt = torch.nn.functional.binary_cross_entropy_with_logits(z, torch.from_numpy(y.astype(np.float64)))
    lt.backward()
    assert abs(lt.item() - loss) <= 1e-12
    for k in P:
        np.testing.assert_allclose(np.asarray(g[k]), T[k].grad.numpy(), rtol=1e-10, atol=1e-13)


def test_zero_hidden_weights_reduce_to_bias_recursion():
    # W1 = W2 = 0, b1 = b2 = 0: h1 = h2 = 0, so only b3 moves: b3 <- b3 - lr (sigmoid(b3) - ybar)
    n, d, h = 30, 4, 3
    X = rng.standard_normal((n, d))
    y = (rng.random(n) < 0.3).astype(np.uint8)
    te = np.zeros(n, bool)
    P0 = dict(W1=np.zeros((h, d)), b1=np.zeros(h), W2=np.zeros((h, h)), b2=np.zeros(h), w3=np.ones(h), b3=0.4)
    P, losses, _ = mlp.train(X, y, te, seed=0, iters=6, lr=0.7, h=h, P0=P0)
    b, ybar = 0.4, y.mean()
    for t in range(6):
        assert abs(losses[t] - (np.logaddexp(0, b) - ybar * b)) <= 1e-14
        b = b - 0.7 * (1 / (1 + np.exp(-b)) - ybar)
    assert abs(P["b3"] - b) <= 1e-14
    np.testing.assert_array_equal(P["W1"], 0)
    np.testing.assert_array_equal(P["w3"], 1)


def test_descent_and_seeded_init():
    n, d, h = 300, 20, 32
    X = rng.standard_normal((n, d))
    y = (X[:, 0] + 0.5 * rng.standard_normal(n) > 0).astype(np.uint8)
    te = np.arange(n) % 5 == 0
    P, losses, met = mlp.train(X, y, te, seed=5, iters=10, lr=0.1, h=h)
    assert np.all(np.diff(losses) < 0)
    assert met["n_train"] + met["n_test"] == n and met["tp"] + met["fp"] + met["tn"] + met["fn"] == met["n_test"]
    P0 = mlp.init_params(5, d, h)
    # bf16-representable, seeded, and the He / LeCun scales of reading R30
    for k in ("W1", "W2", "w3"):
        v = P0[k].astype(np.float32)
        assert np.array_equal(v, torch.from_numpy(v).to(torch.bfloat16).float().numpy())
    assert abs(P0["W1"].std() - np.sqrt(2 / d)) < 0.1 * np.sqrt(2 / d)
    np.testing.assert_array_equal(P0["W2"], mlp.init_params(5, d, h)["W2"])


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _dp_worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    r = np.random.default_rng(11)
    X = r.standard_normal((50, 7))
    y = (r.random(50) < 0.5).astype(np.uint8)
    P = mlp.init_params(9, 7, 6)
    lo, hi = [0, 21, 50][rank], [0, 21, 50][rank + 1]
    # unnormalised gradient sums of this rank's rows = n_shard * mean gradient; allreduce; / n
    _, g = mlp.loss_and_grad(P, X[lo:hi], y[lo:hi])
    flat = np.concatenate([np.ravel(g[k]) * (hi - lo) for k in sorted(g)])
    t = torch.from_numpy(flat.copy())
    dist.all_reduce(t)
    if rank == 0:
        q.put(t.numpy() / 50)
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.timeout(300)
def test_two_rank_data_parallel_gradient_equals_full_batch():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_dp_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    got = q.get(timeout=240)
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    r = np.random.default_rng(11)
    X = r.standard_normal((50, 7))
    y = (r.random(50) < 0.5).astype(np.uint8)
    _, g = mlp.loss_and_grad(mlp.init_params(9, 7, 6), X, y)
    ref = np.concatenate([np.ravel(g[k]) for k in sorted(g)])
    np.testing.assert_allclose(got, ref, rtol=1e-12, atol=1e-15)


def test_standardize_matches_lr_statistics():
    # the MLP's z-scoring is O6 step 2: same mu / population sigma / inv as the C oracle's LR stats pass
    import oracle
    X = rng.standard_normal((60, 9)) * 3 + 1
    X[:, 4] = 0.0   # dead (constant) column -> inv = 0
    te = np.arange(60) % 5 == 0
    mu, sig, inv = oracle.lr_stats(X, te.astype(np.uint8))
    np.testing.assert_allclose(mlp.standardize(X, te), (X - mu) * inv, rtol=1e-13, atol=1e-13)
    assert not mlp.standardize(X, te)[:, 4].any()


def test_bf16_emulation_is_the_definition_up_to_rounding():
    # the diagnostic comparator differs from the fp64 definition only by the bf16 roundings: with the
    # rounding made the identity it must reproduce train() exactly (same algorithm, folded first layer)
    import unittest.mock as um
    n, d, h = 120, 10, 16
    X = np.abs(rng.standard_normal((n, d)))
    y = (rng.random(n) < 0.5).astype(np.uint8)
    te = np.arange(n) % 5 == 0
    R, L, m = mlp.train(X, y, te, seed=3, iters=4, lr=0.05, h=h)
    with um.patch.object(mlp, "_bf16", lambda a: np.asarray(a, dtype=np.float64)):
        E, LE, me = mlp.train_bf16_emulated(X, y, te, seed=3, iters=4, lr=0.05, h=h)
    np.testing.assert_allclose(LE, L, rtol=1e-12)
    for k in ("W1", "W2", "w3", "b1", "b2"):
        np.testing.assert_allclose(E[k], R[k], rtol=1e-9, atol=1e-12)
    assert me["test_acc"] == m["test_acc"] and me["train_acc"] == m["train_acc"]


def test_bf16_budget_covers_bf16_rounding():
    # The a-priori bf16 error budget (tests/mlp_budget.py) that the GPU MLP parity test uses as its tolerance
    # must cover what real bf16 rounding at the product's storage points does: the bf16-emulated algorithm's
    # deviation from the fp64 definition, on real CNN features (AlexNet conv5 / fc6 taps of the oracle).
    import mlp_budget
    from oracle import mlp as M
    tab = gen.make_tables(100, 8)
    F, _ = oracle.features(oracle.ALEXNET, 11, tab.images, taps=[0, 1])
    ps, pi, te = oracle.join(tab.img_keys, tab.str_keys, 5)
    y = tab.labels[ps]
    for t in (0, 1):
        X = oracle.concat(tab.X, F[t], ps, pi)
        B = mlp_budget.budget(X, y, te, seed=21, iters=4, lr=0.01)
        R, lr_, rm = M.train(X, y, te, seed=21, iters=4, lr=0.01)
        E, el, em = M.train_bf16_emulated(X, y, te, seed=21, iters=4, lr=0.01)
        P0 = M.init_params(21, X.shape[1])
        for k in mlp_budget.GROUPS:
            err = np.linalg.norm(E[k] - R[k]) / np.linalg.norm(R[k] - P0[k])
            assert err <= B["upd"][k], (t, k, err, B["upd"][k])
            assert B["upd"][k] < 0.5  # the budget still constrains the update
        assert np.all(np.abs(el - lr_) <= B["loss"])
        assert abs(em["test_acc"] - rm["test_acc"]) <= 100.0 * B["flips"] / rm["n_test"] + 1e-9

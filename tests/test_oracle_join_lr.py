"""Pins of the oracle's join (Eq. (3)), concat (Eq. (4)) and LR (O6).

Join: nested-loop brute force, permutation invariance, primary-key violations.
LR:   central finite differences of the smooth objective; the closed-form first
      gradient at w = 0; ISTA's monotone descent; power iteration on a design
      with a known spectrum; the d = 0 scalar recursion; and convergence to
      scikit-learn's elastic-net logistic regression (saga) on the same
      standardised data — an independent library solver of the same objective.
"""
import numpy as np
import pytest

import gen
import oracle

rng = np.random.default_rng(7)


def brute_join(img_keys, str_keys):
    out = []
    for s, k in enumerate(str_keys):
        for i, kk in enumerate(img_keys):
            if kk == k:
                out.append((s, i))
    return out


@pytest.mark.parametrize("mismatch", [False, True])
def test_join_vs_nested_loop(mismatch):
    t = gen.make_tables(700, 4, mismatch=mismatch, with_images=False)
    ps, pi, te = oracle.join(t.img_keys, t.str_keys, split_seed=9)
    assert list(zip(ps.tolist(), pi.tolist())) == brute_join(t.img_keys.tolist(), t.str_keys.tolist())
    assert len(ps) == (700 - 7 if mismatch else 700)
    # the split flag is a function of the key only
    ss = gen.subseed(9, 6)
    for s, f in zip(ps[:50], te[:50]):
        assert f == (gen.mix64(int(t.str_keys[s]) ^ ss) % 5 == 0)
    assert 0.1 < te.mean() < 0.3


def test_join_permutation_invariance():
    t = gen.make_tables(300, 4, mismatch=True, with_images=False)
    perm = rng.permutation(len(t.img_keys))
    ps, pi, _ = oracle.join(t.img_keys, t.str_keys, 1)
    ps2, pi2, _ = oracle.join(t.img_keys[perm], t.str_keys, 1)
    np.testing.assert_array_equal(ps, ps2)
    np.testing.assert_array_equal(perm[pi2], pi)


def test_join_duplicate_keys():
    k = np.array([5, 6, 7, 6], dtype=np.int64)
    with pytest.raises(oracle.DupKey):
        oracle.join(k, np.array([1], dtype=np.int64), 0)
    with pytest.raises(oracle.DupKey):
        oracle.join(np.array([1, 2]), np.array([2, 3, 2]), 0)


def test_join_empty():
    ps, pi, te = oracle.join(np.zeros(0, dtype=np.int64), np.array([1, 2], dtype=np.int64), 0)
    assert len(ps) == 0


def test_concat_exact_copy():
    X = gen.structured(3, np.arange(6, dtype=np.int64), 3, gen.FOODS)
    F = rng.standard_normal((4, 5))
    ps = np.array([5, 0, 2])
    pi = np.array([1, 3, 0])
    MM = oracle.concat(X, F, ps, pi)
    np.testing.assert_array_equal(MM[:, :3], X[ps].astype(np.float64))
    np.testing.assert_array_equal(MM[:, 3:], F[pi])


def _problem(n=400, d=12, seed=0):
    r = np.random.default_rng(seed)
    X = r.standard_normal((n, d)) * r.uniform(0.5, 3.0, d) + r.uniform(-2, 2, d)
    X[:, 3] = 1.25  # a constant column: sigma = 0, excluded (keep_j = 0)
    logit = X[:, 0] - 0.5 * X[:, 1] + 0.3
    y = (r.uniform(size=n) < 1 / (1 + np.exp(-logit))).astype(np.uint8)
    te = (r.uniform(size=n) < 0.2).astype(np.uint8)
    return X, y, te


def test_lr_stats_population():
    X, y, te = _problem()
    mu, sig, inv = oracle.lr_stats(X, te)
    tr = X[te == 0]
    np.testing.assert_allclose(mu, tr.mean(0), rtol=1e-13, atol=1e-14)
    np.testing.assert_allclose(sig, tr.std(0), rtol=1e-12, atol=1e-14)
    assert inv[3] == 0 and sig[3] == 0


def test_lr_gradient_finite_differences():
    X, y, te = _problem()
    mu, _, inv = oracle.lr_stats(X, te)
    w = rng.standard_normal(X.shape[1]) * 0.3
    b = 0.2
    lam, alpha = 0.01, 0.5
    f, gw, gb = oracle.lr_objective(X, y, te, mu, inv, w, b, lam, alpha)
    h = 1e-6
    for j in range(X.shape[1]):
        e = np.zeros_like(w)
        e[j] = h
        fp = oracle.lr_objective(X, y, te, mu, inv, w + e, b, lam, alpha)[0]
        fm = oracle.lr_objective(X, y, te, mu, inv, w - e, b, lam, alpha)[0]
        fd = (fp - fm) / (2 * h)
        assert abs(fd - gw[j]) <= 1e-6 * max(1.0, abs(gw[j])), j
    fp = oracle.lr_objective(X, y, te, mu, inv, w, b + h, lam, alpha)[0]
    fm = oracle.lr_objective(X, y, te, mu, inv, w, b - h, lam, alpha)[0]
    assert abs((fp - fm) / (2 * h) - gb) <= 1e-6


def test_lr_first_gradient_closed_form():
    # at w = 0, b = 0: g_j = -ybar (mu+_j - mu_j) / sigma_j (mu+ = mean over positive rows)
    X, y, te = _problem()
    mu, sig, inv = oracle.lr_stats(X, te)
    _, gw, gb = oracle.lr_objective(X, y, te, mu, inv, np.zeros(X.shape[1]), 0.0, 0.01, 0.5)
    tr = te == 0
    ybar = y[tr].mean()
    mup = X[tr & (y == 1)].mean(0)
    ref = np.where(sig > 1e-12, -ybar * (mup - mu) / np.where(sig > 0, sig, 1), 0)
    np.testing.assert_allclose(gw, ref, rtol=1e-10, atol=1e-14)
    assert abs(gb - (0.5 - ybar)) < 1e-14


def test_lr_monotone_descent():
    X, y, te = _problem()
    r = oracle.lr_train(X, y, te, iters=30)
    assert np.all(np.diff(r["loss"]) <= 1e-12)
    assert r["loss"][0] == pytest.approx(np.log(2), abs=1e-14)  # z = 0 on the first pass


def test_lr_power_iteration_rank_one():
    # all standardised columns equal (rank 1) + the bias column, centred => spectrum {d_eff, 1}
    n, d = 200, 6
    base = rng.standard_normal(n)
    X = np.repeat(base[:, None], d, axis=1) * np.arange(1, d + 1)  # scaled copies standardise to the same column
    mu, sig, inv = oracle.lr_stats(X, None)
    lam = oracle.lr_power(X, None, mu, inv, 50)
    assert lam == pytest.approx(d, rel=1e-10)


def test_lr_zero_features_scalar_recursion():
    # d = 0 (only the bias): b_{t+1} = b_t - eta (sigmoid(b_t) - ybar), eta = 1 / (0.25 * 1.05 * 1 + lam(1-alpha))
    n = 50
    X = np.zeros((n, 0))
    y = (np.arange(n) % 3 == 0).astype(np.uint8)
    r = oracle.lr_train(X, y, np.zeros(n, np.uint8), iters=4)
    eta = 1.0 / (0.25 * 1.05 * 1.0 + 0.01 * 0.5)
    assert r["eta"] == pytest.approx(eta, rel=1e-14)
    b = 0.0
    for _ in range(4):
        b -= eta * (1 / (1 + np.exp(-b)) - y.mean())
    assert r["b"] == pytest.approx(b, rel=1e-13)


def test_lr_converges_to_sklearn_elastic_net():
    from sklearn.linear_model import LogisticRegression
    X, y, te = _problem(n=300, d=6, seed=3)
    X[:, 3] = X[:, 2] * 0.5 + rng.standard_normal(300)  # no constant column here
    lam, alpha = 0.01, 0.5
    r = oracle.lr_train(X, y, te, iters=20000, lam=lam, alpha=alpha)
    mu, sig, inv = oracle.lr_stats(X, te)
    tr = te == 0
    Z = (X[tr] - mu) * inv
    n = tr.sum()
    sk = LogisticRegression(penalty="elasticnet", solver="saga", l1_ratio=alpha, C=1.0 / (n * lam),
                            fit_intercept=True, tol=1e-12, max_iter=200000)
    sk.fit(Z, y[tr])
    np.testing.assert_allclose(r["w"], sk.coef_[0], atol=2e-4)
    assert r["b"] == pytest.approx(sk.intercept_[0], abs=2e-4)


def test_lr_metrics_vs_sklearn():
    from sklearn.metrics import accuracy_score, f1_score
    X, y, te = _problem()
    r = oracle.lr_train(X, y, te, iters=10)
    mu, _, inv = oracle.lr_stats(X, te)
    z = ((X - mu) * inv) @ r["w"] + r["b"]
    pred = (z >= 0).astype(np.uint8)
    t = te == 1
    assert r["test_acc"] == pytest.approx(100 * accuracy_score(y[t], pred[t]), abs=1e-9)
    assert r["test_f1"] == pytest.approx(100 * f1_score(y[t], pred[t]), abs=1e-9)
    assert r["train_acc"] == pytest.approx(100 * accuracy_score(y[~t], pred[~t]), abs=1e-9)


def test_lr_grad_sums_additive_over_row_shards():
    # the quantity each rank contributes to the allreduce is a sum over its rows
    X, y, te = _problem()
    w = rng.standard_normal(X.shape[1]) * 0.1
    full = oracle.lr_grad_sums(X, y, te, w, 0.1)
    parts = [oracle.lr_grad_sums(X[a:b], y[a:b], te[a:b], w, 0.1) for a, b in [(0, 137), (137, 400)]]
    np.testing.assert_allclose(parts[0] + parts[1], full, rtol=1e-12, atol=1e-12)

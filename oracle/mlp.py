"""Second downstream model M: a 3-layer MLP, plain fp64 numpy (oracle).

TEST INFRASTRUCTURE ONLY (same rule as oracle/__init__.py): only tests/, smoke() and bench.py's
cpu_baseline / reference legs may import it.  Shares no code with the CUDA path; the initial
weights come from the seeded generator in gen/ (vg_param, model id 3).

Paper: "We then train a 3-layer MLP (each hidden layer has 1024 units) for 10 iterations using
distributed TF/Horovod" (§5.1 "Comparing against TF Transform+Beam").
§8f #4.  The paper fixes only the depth, the width and the iteration count; the rest is DESIGN.md
reading R30, stated here step by step:

  x_p   = [X, F_l][p]                       the Eq. (4) row (d = d_s + d_l real columns)
  x~_pj = (x_pj - mu_j) inv_j               z-scored with the train-row statistics of the LR reading
                                            (O6 step 2: population sigma, inv_j = 0 if sigma_j <= 1e-12)
  h1_p  = ReLU(W1 x~_p + b1)                W1: [h, d]
  h2_p  = ReLU(W2 h1_p + b2)                W2: [h, h]
  z_p   = w3 . h2_p + b3                    the third layer: one logit (binary label, as M = LR)
  loss  = (1/n) sum_p [log(1 + e^{z_p}) - y_p z_p]       mean over the n train rows
  T full-batch gradient-descent steps  theta <- theta - lr * grad(loss), lr = 0.01 (the "10 iterations";
  full batch like the LR reading R17, so the result does not depend on the number of GPUs; lr 0.1
  diverged on the synthetic CNN features, whose z-scored covariance has lambda_max ~ 300-900)
  init: W1 ~ N(0, 2/d), W2 ~ N(0, 2/h), w3 ~ N(0, 1/h) (He / LeCun), biases 0, every value rounded
  to bf16 (both sides start from the same numbers); predict 1 iff z >= 0.

Parity status: gradients pinned by central finite differences and by torch autograd (fp64);
the W1 = W2 = 0 special case reduces to the scalar recursion b3 <- b3 - lr (sigmoid(b3) - ybar).
"""
from __future__ import annotations

import numpy as np

import gen

MLP_MODEL_ID = 3  # vg_param "cnn" argument reserved for the downstream MLP's parameters
VG_T_WEIGHT = 0


def init_params(seed: int, d: int, h: int = 1024):
    """Seeded initial parameters (fp64 holding bf16-representable values), reading R30."""
    W1 = gen.param(seed, MLP_MODEL_ID, 0, VG_T_WEIGHT, h * d, 0, 0.0, np.sqrt(2.0 / d), True).reshape(h, d)
    W2 = gen.param(seed, MLP_MODEL_ID, 1, VG_T_WEIGHT, h * h, 0, 0.0, np.sqrt(2.0 / h), True).reshape(h, h)
    w3 = gen.param(seed, MLP_MODEL_ID, 2, VG_T_WEIGHT, h, 0, 0.0, np.sqrt(1.0 / h), True)
    return dict(W1=W1, b1=np.zeros(h), W2=W2, b2=np.zeros(h), w3=w3, b3=0.0)


def _softplus(z):
    return np.logaddexp(0.0, z)


def _sigmoid(z):
    return 0.5 * (1.0 + np.tanh(0.5 * z))


def forward(P, X):
    """h1, h2, z for the rows of X (fp64)."""
    h1 = np.maximum(X @ P["W1"].T + P["b1"], 0.0)
    h2 = np.maximum(h1 @ P["W2"].T + P["b2"], 0.0)
    z = h2 @ P["w3"] + P["b3"]
    return h1, h2, z


def loss_and_grad(P, X, y):
    """Mean logistic loss over the rows of X and its gradient (backpropagation, fp64)."""
    n = X.shape[0]
    y = y.astype(np.float64)
    h1, h2, z = forward(P, X)
    loss = float(np.mean(_softplus(z) - y * z))
    dz = (_sigmoid(z) - y) / n                      # d loss / d z_p
    g = {}
    g["w3"] = h2.T @ dz
    g["b3"] = float(dz.sum())
    dh2 = np.outer(dz, P["w3"]) * (h2 > 0)          # through ReLU
    g["W2"] = dh2.T @ h1
    g["b2"] = dh2.sum(axis=0)
    dh1 = (dh2 @ P["W2"]) * (h1 > 0)
    g["W1"] = dh1.T @ X
    g["b1"] = dh1.sum(axis=0)
    return loss, g


def standardize(X, is_test):
    """x~ = (x - mu) inv with mu, population sigma over the train rows; inv = 0 where sigma <= 1e-12."""
    X = np.asarray(X, dtype=np.float64)
    tr = ~np.asarray(is_test).astype(bool)
    mu = X[tr].mean(axis=0)
    sig = np.sqrt(((X[tr] - mu) ** 2).mean(axis=0))
    inv = np.zeros_like(sig)
    keep = sig > 1e-12
    inv[keep] = 1.0 / sig[keep]
    return (X - mu) * inv


def train(X, y, is_test, seed: int, iters: int = 10, lr: float = 0.01, h: int = 1024, P0=None):
    """T full-batch GD steps on the (z-scored) train rows, then metrics on the test rows (reading R30)."""
    te = np.asarray(is_test).astype(bool)
    X = standardize(X, te)
    y = np.asarray(y).astype(np.uint8)
    Xtr, ytr = X[~te], y[~te]
    P = init_params(seed, X.shape[1], h) if P0 is None else {k: np.array(v, dtype=np.float64) if not np.isscalar(v)
                                                              else float(v) for k, v in P0.items()}
    losses = []
    for _ in range(iters):
        loss, g = loss_and_grad(P, Xtr, ytr)
        losses.append(loss)
        for k in P:
            P[k] = P[k] - lr * g[k]
    _, _, z_tr = forward(P, Xtr)
    _, _, z_te = forward(P, X[te])
    pred_tr = z_tr >= 0
    pred_te = z_te >= 0
    yte = y[te].astype(bool)
    tp = int((pred_te & yte).sum())
    fp = int((pred_te & ~yte).sum())
    fn = int((~pred_te & yte).sum())
    tn = int((~pred_te & ~yte).sum())
    n_te = int(te.sum())
    met = dict(train_acc=100.0 * float((pred_tr == ytr.astype(bool)).mean()) if len(ytr) else 0.0,
               test_acc=100.0 * (tp + tn) / n_te if n_te else 0.0,
               test_f1=100.0 * 2 * tp / (2 * tp + fp + fn) if (2 * tp + fp + fn) else 0.0,
               tp=tp, fp=fp, tn=tn, fn=fn, n_train=int(len(ytr)), n_test=n_te)
    return P, np.array(losses), met


def _bf16(a):
    """Round to the nearest bf16 (RNE) through fp32, returned as fp64."""
    import torch
    return torch.from_numpy(np.asarray(a, dtype=np.float32)).to(torch.bfloat16).to(torch.float64).numpy()


def train_bf16_emulated(X, y, is_test, seed: int, iters: int = 10, lr: float = 0.01, h: int = 1024):
    """DIAGNOSTIC comparator (SURVEY.md §8c c.5 / reading R24 "bf16-emulation mode"), not the definition:
    the same algorithm as train() with the values rounded to bf16 at the points where the B200 path
    stores bf16 (the first layer takes the raw rows with the z-scoring folded into W1' = bf16(W1 diag(inv)),
    b1' = b1 - W1' mu; H1, H2, bf16(W2), dH2, dH2 W2 rounded), everything else in fp64.  It separates
    kernel bugs from bf16 precision drift: the MLP's full-batch gradient at initialisation is a small
    residual of large per-row terms, so 2^-9 roundings of H1 move it by a few percent (measured)."""
    X = np.asarray(X, dtype=np.float64)
    te = np.asarray(is_test).astype(bool)
    y = np.asarray(y).astype(np.uint8)
    tr = ~te
    mu = X[tr].mean(axis=0)
    sig = np.sqrt(((X[tr] - mu) ** 2).mean(axis=0))
    inv = np.zeros_like(sig)
    inv[sig > 1e-12] = 1.0 / sig[sig > 1e-12]
    Xtr, ytr = X[tr], y[tr].astype(np.float64)
    n = Xtr.shape[0]
    P = init_params(seed, X.shape[1], h)
    losses = []

    def fwd(Xr):
        W1b = _bf16(P["W1"] * inv)
        b1p = P["b1"] - W1b @ mu
        h1 = _bf16(np.maximum(Xr @ W1b.T + b1p, 0.0))
        h2 = _bf16(np.maximum(h1 @ _bf16(P["W2"]).T + P["b2"], 0.0))
        return h1, h2, h2 @ P["w3"] + P["b3"]

    for _ in range(iters):
        h1, h2, z = fwd(Xtr)
        losses.append(float(np.mean(_softplus(z) - ytr * z)))
        dz = (_sigmoid(z) - ytr) / n
        dh2 = _bf16(np.outer(dz, P["w3"]) * (h2 > 0))
        dh1 = _bf16(dh2 @ _bf16(P["W2"])) * (h1 > 0)
        g = dict(w3=h2.T @ dz, b3=float(dz.sum()), W2=dh2.T @ h1, b2=dh2.sum(axis=0), b1=dh1.sum(axis=0))
        g["W1"] = (dh1.T @ Xtr - np.outer(g["b1"], mu)) * inv
        for k in P:
            P[k] = P[k] - lr * g[k]
    _, _, z_all = fwd(X)
    pred = z_all >= 0
    yb = y.astype(bool)
    tp = int((pred & yb & te).sum())
    fp = int((pred & ~yb & te).sum())
    fn = int((~pred & yb & te).sum())
    tn = int((~pred & ~yb & te).sum())
    n_te = int(te.sum())
    met = dict(train_acc=100.0 * float((pred[tr] == yb[tr]).mean()) if tr.any() else 0.0,
               test_acc=100.0 * (tp + tn) / n_te if n_te else 0.0, tp=tp, fp=fp, tn=tn, fn=fn,
               n_train=int(tr.sum()), n_test=n_te)
    return P, np.array(losses), met

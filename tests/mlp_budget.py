"""A-priori bf16 error budget of the MLP (reading R30) -- test infrastructure.

The B200 path stores the MLP's activations, back-propagated activations and weight operands in bf16
around fp32-accumulated tcgen05 GEMMs (vista_train_mlp, include/vista.h).  This module predicts, from
the fp64 oracle's own quantities only (never from a GPU result), how far that storage precision can
move the result from the fp64 definition (oracle/mlp.py), with the standard probabilistic model of
rounding error (Higham & Mary): every stored value carries an independent relative error of RMS

    u = 2^-8 / sqrt(6)        (RNE to 8 significant bits: the error is uniform in +-half an ulp =
                               +-2^-8 m for a significand m in [1, 2); E[1/m^2] = 1/2 for uniform m)

and errors are propagated to first order.  fp32 accumulation (2^-24) is negligible next to it.

Storage points (the product's design, R30): h1 = ReLU(W1' x + b1') and h2 in bf16, the
operands W1' = bf16(W1 diag(inv)) and bf16(W2), the back-propagated dH2 and dH1 = bf16(dH2 W2) in bf16.

Per parameter group, the full-batch gradient G = sum_p t_p over the n train rows is a small residual of
large per-row terms (the cancellation the budget has to see): its error is sum_p dt_p with independent
dt_p, so ||dG|| ~ sqrt(sum_p ||dt_p||^2) while ||G|| = ||sum_p t_p||.  Four sources of error:
  backward storage -- the stored factors of t_p (dH2, dH1, h1, h2) and the products dH2 W2, dH1 x;
  forward storage  -- the score z_p shifts by sigma_z,p (h1, h2, W1', W2 stored in bf16), so the
                      residual dz_p = (sigmoid(z_p) - y_p) / n shifts by sigmoid'(z_p) sigma_z,p / n,
                      and every term of the row scales with dz_p;
  shared errors    -- the rounding of a weight OPERAND and the parameter error left by earlier steps are
                      the same for every row, so their effects add coherently over the rows: a matrix
                      times the same signed row sum the gradient is made of;
  ReLU-mask flips  -- a pre-activation within its rounding error of 0 can change sign, which adds or
                      drops a whole term (probability erfc(|a| / (sigma_a sqrt 2)) / 2: the error must
                      point away from a and exceed |a|).
The update after T steps, U = -lr sum_t G_t, is bounded with the triangle inequality over the steps
(eps_U = sum_t ||dG_t|| / ||sum_t G_t||: errors of consecutive steps are correlated, not averaged), and
the parameter error a step leaves behind perturbs the next steps' forward passes (worst case: each
weight row's error aligned with the input it multiplies).
Tolerances are K = 4 standard deviations of that model.
"""
from __future__ import annotations

import numpy as np
from scipy.special import erfc

from oracle import mlp

U = 2.0 ** -8 / np.sqrt(6.0)
K = 4.0
GROUPS = ("W1", "b1", "W2", "b2", "w3")


def _sig(z):
    return 0.5 * (1.0 + np.tanh(0.5 * z))


def _row_budget(P, Xs, y, dev=None):
    """Per-step quantities at parameters P: G, ||dG|| per group, sigma_z per row, loss error RMS.
    dev: per-element RMS deviation of each parameter group accumulated by the previous steps' errors
    (it perturbs this step's forward pass like an extra operand error)."""
    dev = dev or {}
    n = Xs.shape[0]
    W1, W2, w3 = P["W1"], P["W2"], P["w3"]
    dW1, db1, dW2, db2, dw3, db3 = (dev.get(k, 0.0) for k in ("W1", "b1", "W2", "b2", "w3", "b3"))
    h1, h2, z = mlp.forward(P, Xs)
    s = _sig(z)
    r = s - y
    dz = r / n
    sp = s * (1.0 - s)
    m1, m2 = (h1 > 0).astype(np.float64), (h2 > 0).astype(np.float64)
    x2 = (Xs ** 2).sum(axis=1)
    h1n2, h2n2 = (h1 ** 2).sum(axis=1), (h2 ** 2).sum(axis=1)
    W1s, W2s = W1 ** 2, W2 ** 2
    # ---- marginal error variance of every pre-activation / stored value (per row and unit) ----
    va1 = U ** 2 * ((Xs ** 2) @ W1s.T) + dW1 ** 2 * x2[:, None] + db1 ** 2     # W1' operand, deviations
    vh1 = m1 * va1 + U ** 2 * h1 ** 2                                          # + h1 stored
    va2 = vh1 @ W2s.T + U ** 2 * ((h1 ** 2) @ W2s.T) + dW2 ** 2 * h1n2[:, None] + db2 ** 2  # + W2 operand
    vh2 = m2 * va2 + U ** 2 * h2 ** 2                                          # + h2 stored
    # ---- the score: errors propagated linearly (a shared upstream error adds coherently) ----
    g2 = m2 * w3                       # d z / d a2, per row [n, h]
    gh1 = g2 @ W2                      # d z / d h1
    ga1 = gh1 * m1                     # d z / d a1
    var_z = (U ** 2 * (w3 * h2) ** 2).sum(axis=1) + dw3 ** 2 * h2n2 + db3 ** 2
    var_z += (g2 ** 2 * (U ** 2 * ((h1 ** 2) @ W2s.T) + dW2 ** 2 * h1n2[:, None] + db2 ** 2)).sum(axis=1)
    var_z += (gh1 ** 2 * U ** 2 * h1 ** 2).sum(axis=1)
    var_z += (ga1 ** 2 * va1).sum(axis=1)
    sig_z = np.sqrt(var_z)
    dsz = sp * sig_z / n               # RMS shift of dz_p
    # ---- per-row gradient terms and the errors of their factors ----
    dh2 = dz[:, None] * g2             # [n, h]
    dh1 = (dh2 @ W2) * m1
    var_dh1 = m1 * (2.0 * U ** 2 * (dh2 ** 2) @ W2s + dW2 ** 2 * (dh2 ** 2).sum(axis=1)[:, None] + U ** 2 * dh1 ** 2)
    dh2n2 = (dh2 ** 2).sum(axis=1)
    g2n2 = (g2 ** 2).sum(axis=1)
    ga1n2 = (ga1 ** 2).sum(axis=1)
    G = {"W1": dh1.T @ Xs, "b1": dh1.sum(axis=0), "W2": dh2.T @ h1, "b2": dh2.sum(axis=0), "w3": h2.T @ dz}
    back = {"W1": (var_dh1.sum(axis=1) * x2).sum(),
            "b1": var_dh1.sum(),
            "W2": (U ** 2 * dh2n2 * h1n2 + dh2n2 * vh1.sum(axis=1)).sum(),   # dH2 stored; h1's value error
            "b2": U ** 2 * dh2n2.sum(),
            "w3": (dz ** 2 * vh2.sum(axis=1)).sum()}                          # h2's value error
    fwd = {"W1": (dsz ** 2 * ga1n2 * x2).sum(), "b1": (dsz ** 2 * ga1n2).sum(),
           "W2": (dsz ** 2 * g2n2 * h1n2).sum(), "b2": (dsz ** 2 * g2n2).sum(), "w3": (dsz ** 2 * h2n2).sum()}
    # ReLU-mask flips: a pre-activation within its own error of 0 may land on the other side (probability
    # erfc(|a| / (sigma_a sqrt 2)) / 2 for a Gaussian error); a flipped mask adds or drops a whole term
    # dz_p w3_j (layer 2) or (dH2 W2)_pk (layer 1) -- the dominant effect on a gradient that is a small
    # residual of large per-row terms
    a1 = Xs @ W1.T + P["b1"]
    a2 = h1 @ W2.T + P["b2"]
    p1 = 0.5 * erfc(np.abs(a1) / np.sqrt(2.0 * np.maximum(va1, 1e-300)))
    p2 = 0.5 * erfc(np.abs(a2) / np.sqrt(2.0 * np.maximum(va2, 1e-300)))
    f2 = (dz ** 2) * (p2 @ (w3 ** 2))                                   # per row: sum_j P2 (dz w3_j)^2
    f1 = (p1 * (dh2 @ W2) ** 2).sum(axis=1) + (dz ** 2) * ((p2 * w3 ** 2) @ W2s * m1).sum(axis=1)
    flip = {"W1": (f1 * x2).sum(), "b1": f1.sum(), "W2": (f2 * h1n2).sum(), "b2": f2.sum(), "w3": 0.0}
    # the parameter deviations are the SAME for every row, so their effect on a gradient is a matrix times
    # the same signed row sum the gradient itself is made of (its cancellation included):
    #   w3: dG_j = sum_p dz_p m2_pj (dW2_j h1_p + db2_j): per unit j the signed sum v_j = sum_p dz_p m2_pj h1_p
    #       over the rows where unit j is active, with ||dW2_j|| ~ ||dW2|| / sqrt(h)
    #   W2: dG = sum_p dh2_p (dW1 x_p)^T m1     ~ ||sum_p dh2_p x_p^T|| ||dW1||
    aW1, aW2, ab2 = (dev.get("_acc_" + k, 0.0) for k in ("W1", "W2", "b2"))
    coh = {k: 0.0 for k in GROUPS}
    hh = W2.shape[0]
    coh["w3"] = aW2 / np.sqrt(hh) * np.linalg.norm((dz[:, None] * m2).T @ h1) + ab2 / np.sqrt(hh) * np.linalg.norm(dz @ m2)
    coh["W2"] = aW1 * np.linalg.norm(dh2.T @ Xs)
    # the rounding of the W2 OPERAND is also one error shared by every row: for w3 it adds
    # sum_jk dW2_jk V_jk with V = (dz . m2)^T h1, i.e. u ||W2 . V||_F (the dominant w3 term, measured on CPU)
    V2 = (dz[:, None] * m2).T @ h1
    coh["w3"] += U * np.linalg.norm(W2 * V2)
    # ... and it shifts every row's score the same way: the dz shifts add up (worst case, aligned)
    szW = U * np.sqrt((g2 ** 2 * ((h1 ** 2) @ W2s.T)).sum(axis=1))
    dszW = sp * szW / n
    coh["w3"] += (dszW * np.sqrt(h2n2)).sum()
    coh["W2"] += (dszW * np.sqrt(g2n2 * h1n2)).sum()
    coh["b2"] += (dszW * np.sqrt(g2n2)).sum()
    coh["W1"] += (dszW * np.sqrt(ga1n2 * x2)).sum()
    coh["b1"] += (dszW * np.sqrt(ga1n2)).sum()
    dG = {k: np.sqrt(back[k] + fwd[k] + flip[k]) + coh[k] for k in GROUPS}
    loss_rms = np.sqrt(((r * sig_z) ** 2).sum()) / n
    return G, dG, sig_z, z, loss_rms


def budget(X, y, is_test, seed, iters=10, lr=0.01, h=1024):
    """Tolerances for GPU vs fp64 oracle (oracle.mlp.train) on the same rows and initial weights:
    upd[group] (normwise relative error of the update P_T - P_0), loss[t] (absolute), and the number
    of test rows whose prediction may flip (|z| within K standard deviations of its error band)."""
    te = np.asarray(is_test).astype(bool)
    Xs = mlp.standardize(X, te)
    y = np.asarray(y).astype(np.float64)
    Xtr, ytr = Xs[~te], y[~te]
    P = mlp.init_params(seed, X.shape[1], h)
    P0 = {k: (v.copy() if not np.isscalar(v) else v) for k, v in P.items()}
    sumG = {k: 0.0 for k in GROUPS}
    sumdG = {k: 0.0 for k in GROUPS}
    loss_tol = []
    Gn_t, U_t = [], []
    dev = {}
    accum = {k: 0.0 for k in GROUPS}  # norm bound of each group's accumulated parameter error
    for _ in range(iters):
        G, dG, sig_z, _, loss_rms = _row_budget(P, Xtr, ytr, dev)
        Gn_t.append(np.sqrt(sum((G[k] ** 2).sum() for k in GROUPS)))
        U_t.append(np.sqrt(sum(((P[k] - P0[k]) ** 2).sum() for k in GROUPS)))
        for k in GROUPS:
            sumG[k] = sumG[k] + G[k]
            sumdG[k] += dG[k]
            accum[k] += lr * dG[k]
            # worst case: each output unit's weight-row error lies along the input it multiplies (the errors
            # are sums of outer products with those very inputs), so the per-row norm, not a per-element
            # RMS, enters the pre-activations: W1, W2 rows and b1, b2 entries get ||.|| / sqrt(h); w3 whole
            dev[k] = accum[k] / (1.0 if k == "w3" else np.sqrt(np.shape(P[k])[0]))
            dev["_acc_" + k] = accum[k]
        loss_tol.append(K * loss_rms)
        _, g = mlp.loss_and_grad(P, Xtr, ytr)
        for k in P:
            P[k] = P[k] - lr * g[k]
    eps = {k: sumdG[k] / max(np.linalg.norm(sumG[k]), 1e-300) for k in GROUPS}
    eps_max = max(eps.values())
    upd = {k: K * eps[k] for k in GROUPS}
    # the loss at step t also sees the parameter error accumulated before it: |G_t . dU_t|
    loss = np.array([loss_tol[t] + K * eps_max * Gn_t[t] * U_t[t] for t in range(iters)])
    # prediction flips on test rows: band = K sqrt(sigma_z^2 + (eps_U |z_T - z_0|)^2)
    _, _, sig_te, z_te, _ = _row_budget(P, Xs[te], y[te], dev)
    _, _, z0 = mlp.forward(P0, Xs[te])
    band = K * np.sqrt(sig_te ** 2 + (eps_max * (z_te - z0)) ** 2)
    flips = int((np.abs(z_te) <= band).sum())
    return dict(upd=upd, eps=eps, loss=loss, flips=flips, n_test=int(te.sum()))

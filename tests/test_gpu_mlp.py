"""GPU parity of the second downstream model (3-layer MLP; reading R30) through
vista_train_mlp against the fp64 oracle (oracle/mlp.py) on identical inputs: the GPU's own MM_k
rows (bf16, upcast) and the same seeded bf16 initial weights.

Tolerances (R30).  The GPU rounds H1, H2, dH2, dH2 W2 and the weight operands to bf16
(2^-9 relative) around fp32-accumulated tcgen05 GEMMs.  The MLP's full-batch gradient at init is a
small residual of large per-row terms, so those roundings move the weight UPDATE W_T - W_0 by several
percent (reproduced in numpy by oracle.mlp.train_bf16_emulated).  Two comparisons:
  kernels    vs the bf16-emulated algorithm: loss curve <= 1e-3 relative, updates <= 5e-2 normwise
  precision  vs the fp64 definition:         loss curve <= 3e-2 relative, updates <= 0.15 normwise,
             test accuracy within max(0.5 points, 3 test rows) (vs the emulation: one row)
"""
import numpy as np
import pytest
import torch

import gen
from oracle import mlp
from paper_conf_sigmod_nakandalak20_b200 import Vista, VistaError

pytestmark = pytest.mark.gpu
WSEED, SPLIT, MSEED = 11, 5, 21
TOL_LOSS_EMU, TOL_UPD_EMU = 1e-3, 5e-2   # measured on B200: <= 1.7e-4 and <= 2.3e-2
TOL_LOSS_DEF, TOL_UPD_DEF = 3e-2, 0.15    # measured on B200: <= 1.4e-2 and <= 8.5e-2


def gpu_rows(v, k):
    f = v.features(k)
    MM = f["mm"].to(torch.float64).cpu().numpy()
    cols = list(range(f["d_s"])) + list(range(f["ds_pad"], f["ds_pad"] + f["d_l"]))
    X = MM[:, cols]
    y = f["labels"].cpu().numpy()
    te = np.zeros(f["rows"], bool)
    te[f["n_train"]:] = True
    return X, y, te


@pytest.mark.parametrize("cnn,taps,k,n,d_s,iters", [(0, [0, 1], 0, 300, 8, 5), (0, [0, 1], 1, 200, 16, 3),
                                                    (2, [4], 0, 150, 130, 4)])
def test_mlp_vs_oracle_identical_inputs(cnn, taps, k, n, d_s, iters):
    tab = gen.make_tables(n, d_s)
    v = Vista(cnn, layers=taps, n_str_rows=len(tab.str_keys), d_s=d_s, n_images_local=n, iters=2,
              split_seed=SPLIT, weight_seed=WSEED)
    v.transfer(tab.images, tab.img_keys, tab.X, tab.str_keys, tab.labels)
    X, y, te = gpu_rows(v, k)
    P, met = v.train_mlp(k, X.shape[1], iters=iters, lr=0.01, seed=MSEED)
    v.close()
    P0 = mlp.init_params(MSEED, X.shape[1])
    R, losses, rmet = mlp.train(X, y, te, seed=MSEED, iters=iters, lr=0.01)
    E, elosses, emet = mlp.train_bf16_emulated(X, y, te, seed=MSEED, iters=iters, lr=0.01)

    def upd_err(A):
        out = {}
        for name in ("W1", "b1", "W2", "b2", "w3"):
            dref = A[name] - P0[name]
            out[name] = float(np.linalg.norm(P[name] - A[name]) / max(np.linalg.norm(dref), 1e-30))
        return out
    e_emu, e_def = upd_err(E), upd_err(R)
    l_emu = float(np.max(np.abs(np.array(met["loss"]) - elosses) / elosses))
    l_def = float(np.max(np.abs(np.array(met["loss"]) - losses) / losses))
    print("mlp parity", cnn, k, "vs bf16-emulation", e_emu, l_emu, "vs fp64", e_def, l_def,
          met["test_acc"], emet["test_acc"], rmet["test_acc"])
    assert met["n_train"] == rmet["n_train"] and met["n_test"] == rmet["n_test"]
    # kernels: the GPU equals the bf16-emulated algorithm up to fp32-vs-fp64 accumulation
    assert l_emu <= TOL_LOSS_EMU, l_emu
    for name, e in e_emu.items():
        assert e <= TOL_UPD_EMU, (name, e)
    # precision: the fp64 definition, within the measured bf16 drift
    assert l_def <= TOL_LOSS_DEF, l_def
    for name, e in e_def.items():
        assert e <= TOL_UPD_DEF, (name, e)
    one_row = 100.0 / max(rmet["n_test"], 1)
    assert abs(met["test_acc"] - emet["test_acc"]) <= max(0.5, one_row) + 1e-9
    assert abs(met["test_acc"] - rmet["test_acc"]) <= max(0.5, 3 * one_row) + 1e-9


def test_mlp_before_transfer_is_a_state_error():
    v = Vista(0, layers=[1], n_str_rows=4, d_s=8, n_images_local=4)
    with pytest.raises(VistaError) as e:
        v.train_mlp(0, 8 + 4096)
    assert e.value.status == 4
    v.close()

"""fp32 check mode (vista_dtype VISTA_F32, reading R23 in DESIGN.md) against the fp64 oracle.

north_star: features "within a max relative error of 2e-2 for bf16 with fp32 accumulate (1e-4 in
the fp32 check mode)".  Here every layer runs in fp32 storage + fp32 FFMA accumulation, so the
per-image normwise error max|gpu - ref| / max|ref| must be <= 1e-4; the join stays bit-exact and the
LR weights follow the bf16 path's 1e-3 bar (with the oracle LR on the GPU's own fp32 MM, 1e-4).
"""
import numpy as np
import pytest
import torch

import gen
import oracle
from paper_conf_sigmod_nakandalak20_b200 import Vista

pytestmark = pytest.mark.gpu
WSEED = 11
SPLIT = 5
TOL_F32 = 1e-4


def normwise_rows(gpu, ref):
    den = np.maximum(np.abs(ref).max(axis=1), 1e-30)
    return np.abs(gpu - ref).max(axis=1) / den


def oracle_pairs(tab):
    ps, pi, te = oracle.join(tab.img_keys, tab.str_keys, SPLIT)
    order = np.concatenate([np.nonzero(te == 0)[0], np.nonzero(te == 1)[0]])
    return ps[order], pi[order], int((te == 0).sum())


def run_f32(cnn, taps, tab, d_s, iters, **kw):
    v = Vista(cnn, layers=taps, n_str_rows=len(tab.str_keys), d_s=d_s, n_images_local=len(tab.img_keys),
              iters=iters, split_seed=SPLIT, weight_seed=WSEED, dtype="f32", **kw)
    v.transfer(tab.images, tab.img_keys, tab.X, tab.str_keys, tab.labels)
    return v


def test_f32_alexnet_config1_features_join_lr():
    tab = gen.make_tables(16, 8, kind=gen.FOODS)
    taps = [0, 1, 2]
    F, _ = oracle.features(oracle.ALEXNET, WSEED, tab.images, taps=taps)
    v = run_f32(0, taps, tab, 8, iters=5)
    ps, pi, n_train = oracle_pairs(tab)
    y = tab.labels[ps]
    te = np.zeros(len(ps), np.uint8)
    te[n_train:] = 1
    for k, t in enumerate(taps):
        f = v.features(k)
        assert f["features"].dtype == torch.float32 and f["mm"].dtype == torch.float32
        Fg = f["features"].to(torch.float64).cpu().numpy()
        err = normwise_rows(Fg, F[t])
        assert err.max() <= TOL_F32, (t, err.max())
        np.testing.assert_array_equal(f["pair_str"].cpu().numpy(), ps)
        np.testing.assert_array_equal(f["pair_img"].cpu().numpy(), pi)
        MM = f["mm"].to(torch.float64).cpu().numpy()
        np.testing.assert_array_equal(MM[:, :8], tab.X[ps].astype(np.float64))
        np.testing.assert_array_equal(MM[:, f["ds_pad"]:f["ds_pad"] + f["d_l"]], Fg[pi])
        assert not MM[:, f["ds_pad"] + f["d_l"]:].any()
        # LR on identical inputs
        cols = list(range(8)) + list(range(f["ds_pad"], f["ds_pad"] + f["d_l"]))
        ref = oracle.lr_train(MM[:, cols], y, te, iters=5)
        w, b, met = v.train(k, 8 + f["d_l"])
        wr, wg = np.append(ref["w"], ref["b"]), np.append(w, b)
        assert np.linalg.norm(wg - wr) <= 1e-4 * max(np.linalg.norm(wr), 1e-12)
        np.testing.assert_allclose(met["loss"][:5], ref["loss"], rtol=1e-5, atol=1e-7)
        assert met["test_acc"] == ref["test_acc"]
        # end to end: oracle features -> oracle LR
        e2e = oracle.lr_train(oracle.concat(tab.X, F[t], ps, pi), y, te, iters=5)
        we = np.append(e2e["w"], e2e["b"])
        assert np.linalg.norm(wg - we) <= 1e-3 * max(np.linalg.norm(we), 1e-12)
        assert abs(met["test_acc"] - e2e["test_acc"]) <= 0.5 + 1e-9
    v.close()


@pytest.mark.parametrize("plan", ["staged", "eager"])
def test_f32_resnet50_top5(plan):
    tab = gen.make_tables(5, 130, kind=gen.FOODS)
    F, _ = oracle.features(oracle.RESNET50, WSEED, tab.images, taps=[0, 1, 2, 3, 4])
    v = Vista(2, n_top=5, n_str_rows=len(tab.str_keys), d_s=130, n_images_local=5, iters=2, split_seed=SPLIT,
              weight_seed=WSEED, dtype="f32", plan=plan, micro_batch=2)
    v.transfer(tab.images, tab.img_keys, tab.X, tab.str_keys, tab.labels)
    for k in range(5):
        Fg = v.features(k)["features"].to(torch.float64).cpu().numpy()
        err = normwise_rows(Fg, F[k])
        assert err.max() <= TOL_F32, (k, err.max())
    # LR on the widest layer (conv5_x taps: ld = 136 + 8192 fp32 columns)
    w, b, met = v.train(3, 130 + v.features(3)["d_l"])
    assert np.isfinite(w).all() and np.isfinite(b)
    v.close()


def test_f32_vgg16_fc():
    tab = gen.make_tables(2, 201, kind=gen.AMAZON)
    F, _ = oracle.features(oracle.VGG16, WSEED, tab.images, taps=[0, 1, 2])
    v = run_f32(1, [0, 1, 2], tab, 201, iters=2)
    for k in range(3):
        Fg = v.features(k)["features"].to(torch.float64).cpu().numpy()
        assert normwise_rows(Fg, F[k]).max() <= TOL_F32
    v.close()


def test_f32_staged_equals_lazy_bitwise():
    tab = gen.make_tables(6, 8)
    out = {}
    for plan in ("staged", "lazy"):
        v = run_f32(0, [0, 2], tab, 8, iters=2, plan=plan, micro_batch=4)
        out[plan] = [v.features(k)["mm"].cpu().clone() for k in range(2)]
        v.close()
    for a, b in zip(out["staged"], out["lazy"]):
        assert torch.equal(a, b)

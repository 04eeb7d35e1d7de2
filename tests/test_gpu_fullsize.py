"""Full-size parity on the headline path, against the fp64 oracle on the same
generated inputs:

* S4 join: bit-exact at 20k / 200k / 2M keys with unmatched rows on both sides ("Join pairs and
  concat. Bit-exact, full size."), i.e. through the multi-block count / scan / scatter path;
* C2 = BASELINE.json configs[1] (ResNet50 top-5, Foods-shaped, 20,000 images, d_s = 130, T = 10) in
  the launch configuration bench.py times: join and concat bit-exact at full size, features of a
  seeded 64-image subset normwise <= 2e-2 (reading R21), and the LR of every layer (stats, K = 20 power
  iterations, T = 10 ISTA steps, eval; lr_stream_kernel<2> and the ring wrap on the conv5_x layers)
  within 1e-3 of the oracle's O6 run on the GPU's own MM_k (reading R22), loss curve and lambda_hat
  included; the planner's predicted peak against the measured pool high-water mark;
* C1b (parity-only config): AlexNet {conv5, fc6, fc7}, 2,000 images, +-1 % unmatched
  rows, d_s = 8, T = 10: features of every image, and the end-to-end test accuracy and F1 (oracle
  features -> oracle LR vs GPU features -> GPU LR) within a flat 0.5 points.
"""
import concurrent.futures as cf

import numpy as np
import pytest
import torch

import gen
import oracle
from paper_conf_sigmod_nakandalak20_b200 import Vista, VistaError, vista_join

pytestmark = pytest.mark.gpu
SPLIT = 5


def oracle_pairs(img_keys, str_keys):
    ps, pi, te = oracle.join(img_keys, str_keys, SPLIT)
    order = np.concatenate([np.nonzero(te == 0)[0], np.nonzero(te == 1)[0]])  # [train | test], stable
    return ps[order], pi[order], int((te == 0).sum())


def normwise_rows(gpu, ref):
    den = np.maximum(np.abs(ref).max(axis=1), 1e-30)
    return np.abs(gpu - ref).max(axis=1) / den


@pytest.mark.parametrize("N", [20000, 200000, 2000000])
def test_join_full_size_bit_exact(N):
    tab = gen.make_tables(N, 8, mismatch=True, with_images=False)
    ik = torch.from_numpy(tab.img_keys).cuda()
    sk = torch.from_numpy(tab.str_keys).cuda()
    ps, pi, n_train = vista_join(ik, sk, split_seed=SPLIT)
    ops, opi, o_train = oracle_pairs(tab.img_keys, tab.str_keys)
    assert n_train == o_train and len(ps) == len(ops)
    assert len(ops) < len(tab.str_keys) and len(ops) < N  # unmatched rows on both sides
    np.testing.assert_array_equal(ps.cpu().numpy(), ops)
    np.testing.assert_array_equal(pi.cpu().numpy(), opi)
    # permuting T_img permutes the image rows of the pairs and nothing else
    perm = np.random.default_rng(N).permutation(N)
    ps2, pi2, n2 = vista_join(ik[torch.from_numpy(perm).cuda()], sk, split_seed=SPLIT)
    assert n2 == n_train
    np.testing.assert_array_equal(ps2.cpu().numpy(), ops)
    np.testing.assert_array_equal(perm[pi2.cpu().numpy()], opi)  # new image row j holds old row perm[j]
    # a duplicate image key anywhere is a primary-key violation
    ik[N // 2 + 1] = ik[N // 3]
    with pytest.raises(VistaError) as e:
        vista_join(ik, sk, split_seed=SPLIT)
    assert e.value.status == 3


def test_c2_resnet50_foods20k_full_size():
    N, d_s, T = 20000, 130, 10
    tab = gen.make_tables(N, d_s, kind=gen.FOODS)
    v = Vista(2, layers=[0, 1, 2, 3, 4], n_str_rows=N, d_s=d_s, n_images_local=N, iters=T, power_iters=20,
              split_seed=SPLIT, weight_seed=1)
    v.transfer(tab.images, tab.img_keys, tab.X, tab.str_keys, tab.labels)  # host inputs, as bench's e2e
    info = v.plan_info()
    # planner accountability (Eq. (6) analogue): the prediction bounds the measured pool high-water mark
    # and is within 5 % of it
    assert 0 < info["peak_bytes_meas"] <= info["peak_bytes_pred"], info
    assert info["peak_bytes_pred"] - info["peak_bytes_meas"] <= 0.05 * info["peak_bytes_pred"], info
    ps, pi, n_train = oracle_pairs(tab.img_keys, tab.str_keys)
    sub = np.sort(np.random.default_rng(64).choice(N, 64, replace=False))
    Fo, _ = oracle.features(oracle.RESNET50, 1, tab.images[sub], taps=[0, 1, 2, 3, 4])
    ps_t, pi_t = torch.from_numpy(ps).cuda(), torch.from_numpy(pi).cuda()
    X_t = torch.from_numpy(tab.X).cuda().to(torch.bfloat16)
    y = tab.labels[ps]
    te = np.zeros(len(ps), np.uint8)
    te[n_train:] = 1
    gpu, inputs = [], []
    for k in range(5):
        f = v.features(k)
        assert f["rows"] == len(ps) and f["n_train"] == n_train
        assert np.array_equal(f["pair_str"].cpu().numpy(), ps) and np.array_equal(f["pair_img"].cpu().numpy(), pi)
        assert np.array_equal(f["labels"].cpu().numpy(), y)
        mm, F = f["mm"], f["features"]
        ds_pad, d_l = f["ds_pad"], f["d_l"]
        # concat (Eq. 4): an exact copy, full size
        assert torch.equal(mm[:, :d_s].view(torch.int16), X_t[ps_t.long()].view(torch.int16))
        assert not mm[:, d_s:ds_pad].view(torch.int16).any()
        assert torch.equal(mm[:, ds_pad:ds_pad + d_l].view(torch.int16), F[pi_t.long()].view(torch.int16))
        assert not mm[:, ds_pad + d_l:].view(torch.int16).any()
        # features: normwise per image on the seeded subset
        err = normwise_rows(F[torch.from_numpy(sub).cuda()].double().cpu().numpy(), Fo[k])
        assert err.max() <= 2e-2, (k, err.max())
        gpu.append(v.train(k, d_s + d_l))
        inputs.append((k, ds_pad, d_l))
    mms = [v.features(k)["mm"] for k in range(5)]

    def oracle_lr(arg):
        k, ds_pad, d_l = arg
        cols = torch.cat([torch.arange(d_s), torch.arange(ds_pad, ds_pad + d_l)]).cuda()
        X = mms[k][:, cols].double().cpu().numpy()
        return oracle.lr_train(X, y, te, iters=T)

    with cf.ThreadPoolExecutor(5) as ex:  # the oracle releases the GIL (ctypes)
        refs = list(ex.map(oracle_lr, inputs))
    for k in range(5):
        w, b, met = gpu[k]
        ref = refs[k]
        wr, wg = np.append(ref["w"], ref["b"]), np.append(w, b)
        rel = np.linalg.norm(wg - wr) / np.linalg.norm(wr)
        assert rel <= 1e-3, (k, rel)
        np.testing.assert_allclose(met["loss"][:T], ref["loss"], rtol=1e-4, atol=1e-6)
        assert met["lambda_hat"] == pytest.approx(ref["lambda_hat"], rel=1e-4)
        assert met["n_train"] == ref["n_train"] and met["n_test"] == ref["n_test"]
        assert abs(met["test_acc"] - ref["test_acc"]) <= 0.5, (k, met["test_acc"], ref["test_acc"])
        assert abs(met["train_acc"] - ref["train_acc"]) <= 0.5
    v.close()


def test_c1b_alexnet_2000_end_to_end_accuracy():
    N, d_s, T, taps = 2000, 8, 10, [0, 1, 2]
    tab = gen.make_tables(N, d_s, mismatch=True)
    Fo, _ = oracle.features(oracle.ALEXNET, 11, tab.images, taps=taps)
    ps, pi, n_train = oracle_pairs(tab.img_keys, tab.str_keys)
    assert len(ps) < len(tab.str_keys) and len(ps) < N  # +-1 % unmatched on both sides
    y = tab.labels[ps]
    te = np.zeros(len(ps), np.uint8)
    te[n_train:] = 1
    res = {}
    for plan in ("staged", "eager", "lazy"):
        v = Vista(0, layers=taps, n_str_rows=len(tab.str_keys), d_s=d_s, n_images_local=N, iters=T,
                  split_seed=SPLIT, weight_seed=11, plan=plan)
        v.transfer(tab.images, tab.img_keys, tab.X, tab.str_keys, tab.labels)
        res[plan] = [v.features(k)["mm"].view(torch.int16).cpu().clone() for k in range(3)]
        if plan != "staged":
            v.close()
            continue
        for k, t in enumerate(taps):
            f = v.features(k)
            assert np.array_equal(f["pair_str"].cpu().numpy(), ps) and np.array_equal(f["pair_img"].cpu().numpy(), pi)
            Fg = f["features"].double().cpu().numpy()
            assert normwise_rows(Fg, Fo[t]).max() <= 2e-2  # every image
            w, b, met = v.train(k, d_s + f["d_l"])
            # end to end: oracle features -> oracle concat -> oracle LR (Eqs. (2)-(4) in fp64)
            e2e = oracle.lr_train(oracle.concat(tab.X, Fo[t], ps, pi), y, te, iters=T)
            assert met["n_test"] == e2e["n_test"] and met["n_test"] >= 350
            assert abs(met["test_acc"] - e2e["test_acc"]) <= 0.5, (k, met["test_acc"], e2e["test_acc"])
            assert abs(met["test_f1"] - e2e["test_f1"]) <= 0.5, (k, met["test_f1"], e2e["test_f1"])
        v.close()
    for plan in ("eager", "lazy"):
        for a, b in zip(res["staged"], res[plan]):
            assert torch.equal(a, b), plan

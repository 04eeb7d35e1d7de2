"""Pins of the oracle's network forward passes.

1. An independent implementation of each roster CNN composed only of torch
   library routines (conv2d, batch_norm, local_response_norm, max_pool2d,
   linear) in fp64, fed with the same generated parameters (gen.param) under
   its own shape bookkeeping, must reproduce every tap.
2. The Staged invariant (§5.2, "All approaches ... yield identical
   downstream models"): staged (continue from the stored tap activation, Fig 5E)
   == eager (one pass tapping all layers, Fig 5C) == lazy (recompute from pixels
   per layer, Fig 5A), exactly in fp64.
"""
import numpy as np
import pytest
import torch
import torch.nn.functional as Fn

import gen
import oracle

SEED = 77


def P(cnn, layer, tensor, n, kind, mean, std, rnd):
    return torch.from_numpy(gen.param(SEED, cnn, layer, tensor, n, kind, mean, std, rnd))


def conv_w(cnn, lid, cout, k, cin_g):
    fan = k * k * cin_g
    w = P(cnn, lid, 0, cout * fan, 0, 0.0, (2.0 / fan) ** 0.5, True).reshape(cout, k, k, cin_g)
    return w.permute(0, 3, 1, 2).contiguous()  # OHWI -> OIHW


def bias(cnn, lid, n):
    return P(cnn, lid, 1, n, 0, 0.0, 0.01, True)


def fc_w(cnn, lid, nout, nin):
    return P(cnn, lid, 0, nout * nin, 0, 0.0, (2.0 / nin) ** 0.5, True).reshape(nout, nin)


def nhwc_flat(x):
    return x.permute(0, 2, 3, 1).reshape(x.shape[0], -1)


def tap2x2(a):
    H = a.shape[-1]
    k = (H + 1) // 2
    return nhwc_flat(Fn.max_pool2d(a, k, k, ceil_mode=True))


def pixels(imgs):
    return (torch.from_numpy(imgs.astype(np.float64)) - 128.0).div(128.0).permute(0, 3, 1, 2)


def torch_alexnet(imgs):
    c = 0
    x = pixels(imgs)
    spec = [(96, 11, 3, 1, 4, 0), (256, 5, 96, 2, 1, 2), (384, 3, 256, 1, 1, 1), (384, 3, 384, 2, 1, 1),
            (256, 3, 384, 2, 1, 1)]
    for lid, (co, k, ci, g, s, p) in enumerate(spec):
        x = Fn.relu(Fn.conv2d(x, conv_w(c, lid, co, k, ci // g), bias(c, lid, co), stride=s, padding=p, groups=g))
        if lid < 2:
            x = Fn.max_pool2d(Fn.local_response_norm(x, 5, alpha=1e-4, beta=0.75, k=1.0), 3, 2)
    taps = [tap2x2(x)]
    x = nhwc_flat(Fn.max_pool2d(x, 3, 2))
    x = Fn.relu(Fn.linear(x, fc_w(c, 5, 4096, 9216), bias(c, 5, 4096)))
    taps.append(x)
    x = Fn.relu(Fn.linear(x, fc_w(c, 6, 4096, 4096), bias(c, 6, 4096)))
    taps.append(x)
    taps.append(Fn.linear(x, fc_w(c, 7, 1000, 4096), bias(c, 7, 1000)))
    return [t.numpy() for t in taps]


def bn(x, cnn, lid, n, last):
    g = P(cnn, lid, 2, n, 0, 0.2, 0.02, False) if last else P(cnn, lid, 2, n, 0, 1.0, 0.1, False)
    b = P(cnn, lid, 3, n, 0, 0.0, 0.05, False)
    m = P(cnn, lid, 4, n, 0, 0.0, 0.05, False)
    v = P(cnn, lid, 5, n, 1, 1.0, 0.2, False)
    return Fn.batch_norm(x, m, v, g, b, training=False, eps=1e-5)


def torch_resnet50(imgs):
    c = 2
    x = pixels(imgs)
    x = Fn.relu(bn(Fn.conv2d(x, conv_w(c, 0, 64, 7, 3), stride=2, padding=3), c, 0, 64, False))
    x = Fn.max_pool2d(x, 3, 2)
    lid, cin, taps = 1, 64, []
    for st, (mid, units) in enumerate([(64, 3), (128, 4), (256, 6), (512, 3)]):
        for u in range(units):
            s = 2 if (u == 0 and st > 0) else 1
            a = Fn.relu(bn(Fn.conv2d(x, conv_w(c, lid, mid, 1, cin), stride=s), c, lid, mid, False))
            b = Fn.relu(bn(Fn.conv2d(a, conv_w(c, lid + 1, mid, 3, mid), padding=1), c, lid + 1, mid, False))
            y = bn(Fn.conv2d(b, conv_w(c, lid + 2, 4 * mid, 1, mid)), c, lid + 2, 4 * mid, True)
            if u == 0:
                sc = bn(Fn.conv2d(x, conv_w(c, lid + 3, 4 * mid, 1, cin), stride=s), c, lid + 3, 4 * mid, True)
                lid += 4
            else:
                sc = x
                lid += 3
            x = Fn.relu(y + sc)
            cin = 4 * mid
            if (st == 2 and u == 5) or st == 3:
                taps.append(tap2x2(x))
    assert lid == 53
    x = x.mean(dim=(2, 3))
    taps.append(Fn.linear(x, fc_w(c, 53, 1000, 2048), bias(c, 53, 1000)))
    return [t.numpy() for t in taps]


def torch_vgg16(imgs):
    # configuration D of [61] at 227 (reading R1): 13 conv3x3 pad 1 + bias + ReLU, 2x2/2 max pools after
    # convs 2, 4, 7, 10, 13 (227 -> 113 -> 56 -> 28 -> 14 -> 7), NHWC flatten (reading R8) -> fc6 -> fc7 -> fc8
    c = 1
    x = pixels(imgs)
    chans = [64, 64, 128, 128, 256, 256, 256, 512, 512, 512, 512, 512, 512]
    pool_after = {1, 3, 6, 9, 12}
    cin = 3
    for lid, co in enumerate(chans):
        x = Fn.relu(Fn.conv2d(x, conv_w(c, lid, co, 3, cin), bias(c, lid, co), padding=1))
        if lid in pool_after:
            x = Fn.max_pool2d(x, 2, 2)
        cin = co
    assert tuple(x.shape[1:]) == (512, 7, 7)
    x = nhwc_flat(x)
    fc6 = Fn.relu(Fn.linear(x, fc_w(c, 13, 4096, 25088), bias(c, 13, 4096)))
    fc7 = Fn.relu(Fn.linear(fc6, fc_w(c, 14, 4096, 4096), bias(c, 14, 4096)))
    fc8 = Fn.linear(fc7, fc_w(c, 15, 1000, 4096), bias(c, 15, 1000))
    return [t.numpy() for t in (fc6, fc7, fc8)]


@pytest.fixture(scope="module")
def imgs():
    t = gen.make_tables(3, 8, seed=gen.DEFAULT_SEED)
    return t.images[:2]


def _close(a, b):
    scale = np.abs(b).max()
    return np.abs(a - b).max() <= 1e-10 * max(scale, 1.0)


def test_alexnet_vs_torch_library(imgs):
    F, _ = oracle.features(oracle.ALEXNET, SEED, imgs, taps=[0, 1, 2, 3])
    ref = torch_alexnet(imgs)
    for t in range(4):
        assert _close(F[t], ref[t]), t


@pytest.mark.slow
def test_resnet50_vs_torch_library(imgs):
    F, _ = oracle.features(oracle.RESNET50, SEED, imgs[:1], taps=[0, 1, 2, 3, 4])
    ref = torch_resnet50(imgs[:1])
    for t in range(5):
        assert _close(F[t], ref[t]), t


@pytest.mark.slow
def test_vgg16_vs_torch_library(imgs):
    # pins the oracle's VGG16 composition (ReLUs, biases, pool positions, the fc6 flatten order) against
    # torch library routines on the same generated parameters, not only its MAC total and tap widths
    F, _ = oracle.features(oracle.VGG16, SEED, imgs[:1], taps=[0, 1, 2])
    ref = torch_vgg16(imgs[:1])
    for t in range(3):
        assert _close(F[t], ref[t]), t
        assert np.abs(ref[t]).max() > 1e-3  # the activations did not collapse to zero


def test_staged_eager_lazy_alexnet(imgs):
    cnn = oracle.ALEXNET
    T = oracle.n_taps(cnn)
    eager, acts = oracle.features(cnn, SEED, imgs, taps=list(range(T)), want_act=list(range(T)))
    # staged: stage k continues from the stored activation of stage k-1 (Fig 5E)
    for t in range(1, T):
        Ft, _ = oracle.features_from(cnn, SEED, t - 1, acts[t - 1], taps=[t])
        np.testing.assert_array_equal(Ft[t], eager[t])
    # lazy: every layer recomputed from raw pixels (Fig 5A)
    for t in range(T):
        Ft, _ = oracle.features(cnn, SEED, imgs, taps=[t])
        np.testing.assert_array_equal(Ft[t], eager[t])


def test_thread_count_invariance(imgs):
    a, _ = oracle.features(oracle.ALEXNET, SEED, imgs, taps=[0], nthreads=1)
    b, _ = oracle.features(oracle.ALEXNET, SEED, imgs, taps=[0], nthreads=2)
    np.testing.assert_array_equal(a[0], b[0])

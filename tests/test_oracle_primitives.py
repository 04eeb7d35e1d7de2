"""Pins of the oracle's primitives against library routines and brute force
(DESIGN.md §"Oracle pins").  CPU only."""
import itertools

import numpy as np
import pytest
import torch
import torch.nn.functional as Fn

import oracle

rng = np.random.default_rng(1234)


def _torch_conv(x, w, stride, pad, groups, bias=None):
    xt = torch.from_numpy(x).permute(0, 3, 1, 2)              # NCHW
    wt = torch.from_numpy(w).permute(0, 3, 1, 2)              # O, C/g, R, S
    bt = torch.from_numpy(bias) if bias is not None else None
    return Fn.conv2d(xt, wt, bt, stride=stride, padding=pad, groups=groups).permute(0, 2, 3, 1).numpy()


def _im2col_conv(x, w, stride, pad, groups):
    """An independent formulation: explicit zero-padded im2col + matmul per group."""
    N, H, W, C = x.shape
    Cout, R, S, Cg = w.shape
    xp = np.zeros((N, H + 2 * pad, W + 2 * pad, C))
    xp[:, pad:pad + H, pad:pad + W, :] = x
    Ho, Wo = (H + 2 * pad - R) // stride + 1, (W + 2 * pad - S) // stride + 1
    y = np.zeros((N, Ho, Wo, Cout))
    Cog = Cout // groups
    for g in range(groups):
        cols = np.zeros((N, Ho, Wo, R, S, Cg))
        for r in range(R):
            for s in range(S):
                cols[:, :, :, r, s, :] = xp[:, r:r + stride * Ho:stride, s:s + stride * Wo:stride, g * Cg:(g + 1) * Cg]
        wg = w[g * Cog:(g + 1) * Cog].reshape(Cog, -1)
        y[..., g * Cog:(g + 1) * Cog] = cols.reshape(N, Ho, Wo, -1) @ wg.T
    return y


CONV_CASES = [
    # k, stride, pad, groups, C, Cout, H
    (1, 1, 0, 1, 8, 6, 5), (1, 2, 0, 1, 8, 4, 7), (3, 1, 1, 1, 4, 8, 6), (3, 1, 1, 2, 8, 4, 5),
    (3, 2, 1, 1, 3, 5, 9), (5, 1, 2, 2, 4, 6, 7), (7, 2, 3, 1, 3, 4, 9), (11, 4, 0, 1, 3, 4, 15),
    (3, 4, 0, 1, 2, 3, 9), (5, 2, 0, 2, 6, 4, 9), (1, 1, 0, 4, 8, 8, 3),
]


@pytest.mark.parametrize("k,stride,pad,groups,C,Cout,H", CONV_CASES)
def test_conv2d_vs_torch_and_im2col(k, stride, pad, groups, C, Cout, H):
    x = rng.standard_normal((2, H, H + 1, C))
    w = rng.standard_normal((Cout, k, k, C // groups))
    b = rng.standard_normal(Cout)
    y = oracle.conv2d(x, w, stride, pad, groups, bias=b)
    np.testing.assert_allclose(y, _torch_conv(x, w, stride, pad, groups, b), rtol=1e-12, atol=1e-12)
    y0 = oracle.conv2d(x, w, stride, pad, groups)
    np.testing.assert_allclose(y0, _im2col_conv(x, w, stride, pad, groups), rtol=1e-12, atol=1e-12)


def test_conv2d_brute_force_single_output():
    # one output element by the defining sum, written as a literal loop over the window
    x = rng.standard_normal((1, 5, 5, 2))
    w = rng.standard_normal((3, 3, 3, 2))
    y = oracle.conv2d(x, w, stride=2, pad=1)
    ho, wo, o = 1, 2, 1
    acc = 0.0
    for r, s, c in itertools.product(range(3), range(3), range(2)):
        hi, wi = ho * 2 - 1 + r, wo * 2 - 1 + s
        if 0 <= hi < 5 and 0 <= wi < 5:
            acc += x[0, hi, wi, c] * w[o, r, s, c]
    assert abs(y[0, ho, wo, o] - acc) < 1e-13


def test_fc_vs_matmul():
    x = rng.standard_normal((3, 17))
    w = rng.standard_normal((5, 17))
    b = rng.standard_normal(5)
    np.testing.assert_allclose(oracle.fc(x, w, b), x @ w.T + b, rtol=1e-13, atol=1e-13)
    np.testing.assert_allclose(oracle.fc(x, w), Fn.linear(torch.from_numpy(x), torch.from_numpy(w)).numpy(),
                               rtol=1e-13, atol=1e-13)


@pytest.mark.parametrize("k,s,H", [(3, 2, 13), (3, 2, 114), (2, 2, 227), (2, 2, 7), (3, 2, 55), (3, 2, 8)])
def test_maxpool_vs_torch(k, s, H):
    x = rng.standard_normal((2, H, H, 3))
    ref = Fn.max_pool2d(torch.from_numpy(x).permute(0, 3, 1, 2), k, s).permute(0, 2, 3, 1).numpy()
    np.testing.assert_array_equal(oracle.maxpool(x, k, s), ref)


def test_avgpool_vs_mean():
    x = rng.standard_normal((2, 7, 7, 5))
    np.testing.assert_allclose(oracle.avgpool_global(x), x.mean(axis=(1, 2)), rtol=1e-14)


def test_lrn_vs_torch():
    x = rng.standard_normal((2, 4, 3, 11)) * 30  # large enough that the normaliser matters
    ref = Fn.local_response_norm(torch.from_numpy(x).permute(0, 3, 1, 2), size=5, alpha=1e-4, beta=0.75, k=1.0)
    np.testing.assert_allclose(oracle.lrn(x), ref.permute(0, 2, 3, 1).numpy(), rtol=1e-12, atol=1e-14)


def test_batchnorm_vs_torch():
    x = rng.standard_normal((2, 3, 3, 6))
    g, b, m = rng.standard_normal(6), rng.standard_normal(6), rng.standard_normal(6)
    v = rng.uniform(0.5, 2.0, 6)
    ref = Fn.batch_norm(torch.from_numpy(x).permute(0, 3, 1, 2), torch.from_numpy(m), torch.from_numpy(v),
                        torch.from_numpy(g), torch.from_numpy(b), training=False, eps=1e-5)
    np.testing.assert_allclose(oracle.batchnorm(x, g, b, m, v), ref.permute(0, 2, 3, 1).numpy(), rtol=1e-12,
                               atol=1e-13)


@pytest.mark.parametrize("H,W,C", [(14, 14, 16), (7, 7, 8), (13, 13, 4), (2, 2, 3), (3, 5, 2), (1, 1, 4)])
def test_tap_closed_form_on_ramp(H, W, C):
    # A[h,w,c] = (h W + w) C + c is increasing in h and w, so the max of each
    # quadrant sits at its last row/column: R_0 = [0, ceil(H/2)), R_1 = [ceil(H/2), H).
    A = np.arange(H * W * C, dtype=np.float64).reshape(1, H, W, C)
    F = oracle.tap(A).reshape(2, 2, C)
    h2, w2 = (H + 1) // 2, (W + 1) // 2
    last_h = [h2 - 1, H - 1]
    last_w = [w2 - 1, W - 1]
    for i in range(2):
        for j in range(2):
            if H == 1 and i == 1 or W == 1 and j == 1:
                continue  # empty quadrant for a 1-wide side
            np.testing.assert_array_equal(F[i, j], A[0, last_h[i], last_w[j]])


@pytest.mark.parametrize("H", [14, 7, 13])
def test_tap_vs_torch_ceil_maxpool(H):
    # reading R7 = torch max_pool2d with kernel = stride = ceil(H/2), ceil_mode (window truncated)
    C = 6
    A = rng.standard_normal((3, H, H, C))
    k = (H + 1) // 2
    ref = Fn.max_pool2d(torch.from_numpy(A).permute(0, 3, 1, 2), k, k, ceil_mode=True)
    assert ref.shape[-2:] == (2, 2)
    ref = ref.permute(0, 2, 3, 1).reshape(3, 4 * C).numpy()  # NHWC flatten: (2i + j) C + c
    np.testing.assert_array_equal(oracle.tap(A), ref)

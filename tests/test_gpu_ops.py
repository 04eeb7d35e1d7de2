"""GPU parity of single kernels (through the C-ABI kernel-level entry points) against
the fp64 oracle on identical bf16-valued inputs.

Tolerance (DESIGN.md §"Tolerances"): a conv/FC output is fp32-accumulated and rounded
once to bf16 (RNE, relative 2^-9); normwise max|gpu - ref| / max|ref| <= 8e-3 leaves
margin for fp32 summation order.  Max-based ops (tap, max pool) are bit-exact.
"""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_sigmod_nakandalak20_b200 import (vista_avgpool, vista_conv2d, vista_ingest, vista_lrn,
                                                 vista_maxpool, vista_tap)

pytestmark = pytest.mark.gpu
rng = np.random.default_rng(2020)


def bf(a):
    """numpy float -> (bf16 cuda tensor, the same values as fp64 numpy)."""
    t = torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32)).to(torch.bfloat16)
    return t.cuda(), t.to(torch.float64).numpy()


def normwise(gpu, ref):
    return float(np.abs(gpu - ref).max() / max(np.abs(ref).max(), 1e-30))


CONV = [
    # N, H, W, C, Cout, k, stride, pad, groups, residual, relu     (what it covers)
    (2, 14, 14, 64, 256, 1, 1, 0, 1, True, True),      # 1x1 s1 (fast path), BN=256, residual
    (2, 14, 14, 256, 128, 1, 2, 0, 1, False, True),    # 1x1 s2 projection-style, BN=128
    (2, 9, 11, 64, 64, 3, 1, 1, 1, False, True),       # 3x3 p1, BN=64, M tail (198 rows)
    (1, 23, 23, 8, 64, 7, 2, 3, 1, False, True),       # conv1-style 7x7 s2, C=8 (general gather)
    (1, 31, 31, 8, 96, 11, 4, 0, 1, False, True),      # AlexNet conv1 geometry, Cout 96 (masked N tile)
    (1, 9, 9, 96, 256, 5, 1, 2, 2, False, True),       # grouped 5x5, Cg_in = 48 (general gather)
    (1, 7, 7, 384, 384, 3, 1, 1, 2, False, True),      # grouped 3x3, Cg_out = 192
    (3, 1, 1, 1152, 1000, 1, 1, 0, 1, False, False),   # FC, N = 1000 (partial last N tile), M = 3
    (2, 7, 7, 128, 512, 3, 2, 1, 1, True, False),      # strided 3x3, residual without ReLU
    (130, 1, 1, 64, 128, 1, 1, 0, 1, False, True),     # FC with M = 130 (two M tiles)
    (2, 17, 17, 8, 64, 3, 1, 1, 1, False, True),       # VGG conv1_1-style, row-gather mode
    (1, 9, 9, 96, 96, 3, 1, 1, 2, True, True),         # Cg_out = 48: masked group tile, register epilogue
    (2, 15, 15, 64, 256, 1, 1, 0, 1, True, True),      # TMA A + TMA epilogue, M tail (450 rows), residual
    (3, 1, 1, 2048, 1000, 1, 1, 0, 1, True, False),    # FC 1000 with BN = 256 partial tile + residual
    (2, 20, 23, 16, 64, 4, 1, 0, 1, False, True),      # space-to-depth conv1 shape: TMA row view (Wo = 20)
    (1, 12, 12, 16, 64, 4, 1, 0, 1, True, True),       # same class with residual: row gather fallback
    (2, 56, 56, 64, 64, 3, 1, 1, 1, False, True),      # ResNet res2 3x3: halo mode (Wp = 58), BN = 64
    (3, 28, 28, 128, 128, 3, 1, 1, 1, False, True),    # ResNet res3 3x3: halo mode, BN = 128, 2 channel blocks
    (2, 10, 10, 128, 64, 3, 1, 1, 1, False, False),    # halo mode, tiles spanning image ends, no ReLU
    (1, 5, 130, 64, 64, 3, 1, 1, 1, False, True),      # wide rows: halo does not fit -> im2col boxes
    (7, 56, 56, 64, 64, 3, 1, 1, 1, False, True),      # halo + resident weights (>= 148 tiles), 3 halo buffers
    (13, 14, 14, 256, 1024, 1, 1, 0, 1, True, True),   # 1x1 resident weights, 8 N tiles (grid 144), M tail
    (6, 28, 28, 128, 512, 1, 1, 0, 1, False, True),    # 1x1 resident weights, K = 128, 4 N tiles
    (24, 28, 28, 128, 128, 3, 1, 1, 1, True, True),    # res3 3x3 on the CTA pair (cta_group::2, M = 256), residual
    (23, 28, 28, 128, 128, 3, 1, 1, 1, False, True),   # CTA pair with an odd image count: phantom rank-1 tiles
    (101, 14, 14, 256, 256, 3, 1, 1, 1, True, True),   # res4 3x3 on the CTA pair (im2col, M = N = 256), phantom tile
]


@pytest.mark.parametrize("N,H,W,C,Cout,k,stride,pad,groups,residual,relu", CONV)
def test_conv_tcgen05_vs_oracle(N, H, W, C, Cout, k, stride, pad, groups, residual, relu):
    x, x64 = bf(rng.standard_normal((N, H, W, C)))
    w, w64 = bf(rng.standard_normal((Cout, k, k, C // groups)) * (2.0 / (k * k * C / groups)) ** 0.5)
    scale = rng.uniform(0.5, 1.5, Cout).astype(np.float32)
    shift = rng.standard_normal(Cout).astype(np.float32) * 0.1
    ref = oracle.conv2d(x64, w64, stride, pad, groups) * scale.astype(np.float64) + shift.astype(np.float64)
    res = None
    if residual:
        res, res64 = bf(rng.standard_normal(ref.shape))
        ref = ref + res64
    if relu:
        ref = np.maximum(ref, 0)
    y = vista_conv2d(x, w, torch.from_numpy(scale).cuda(), torch.from_numpy(shift).cuda(), stride, pad, groups,
                     residual=res, relu=relu)
    torch.cuda.synchronize()
    got = y.to(torch.float64).cpu().numpy()
    assert got.shape == ref.shape
    assert normwise(got, ref) <= 8e-3


def test_conv_deterministic():
    x, _ = bf(rng.standard_normal((2, 14, 14, 64)))
    w, _ = bf(rng.standard_normal((128, 3, 3, 64)) * 0.05)
    s = torch.ones(128, device="cuda")
    b = torch.zeros(128, device="cuda")
    y1 = vista_conv2d(x, w, s, b, 1, 1)
    y2 = vista_conv2d(x, w, s, b, 1, 1)
    assert torch.equal(y1.view(torch.int16), y2.view(torch.int16))


@pytest.mark.parametrize("N,H,C,Cout,res", [(3, 14, 256, 1024, True), (5, 7, 512, 2048, True), (2, 9, 64, 128, False),
                                            (4, 13, 128, 256, False),
                                            (64, 7, 512, 2048, True),     # CTA-pair launch (cg2), phantom tile
                                            (97, 14, 256, 1024, True)])   # resident weights, many tiles
def test_fused_tap_bit_exact(N, H, C, Cout, res):
    # the conv4_6 / conv5_x producers: 1x1 convs with residual + ReLU; the tap fused into the epilogue
    # must equal the standalone tap of the same bf16 output bit for bit (max is exact), and the oracle's
    from paper_conf_sigmod_nakandalak20_b200.vista import vista_conv2d_tap
    x, _ = bf(rng.standard_normal((N, H, H, C)))
    w, _ = bf(rng.standard_normal((Cout, 1, 1, C)) * (2.0 / C) ** 0.5)
    scale = torch.from_numpy(rng.uniform(0.5, 1.5, Cout).astype(np.float32)).cuda()
    shift = torch.from_numpy((rng.standard_normal(Cout) * 0.1).astype(np.float32)).cuda()
    r = bf(rng.standard_normal((N, H, H, Cout)))[0] if res else None
    y, F = vista_conv2d_tap(x, w, scale, shift, residual=r)
    y2 = vista_conv2d(x, w, scale, shift, residual=r, relu=True)
    assert torch.equal(y.view(torch.int16), y2.view(torch.int16))
    assert torch.equal(F.view(torch.int16), vista_tap(y).view(torch.int16))
    np.testing.assert_array_equal(F.to(torch.float64).cpu().numpy(), oracle.tap(y.to(torch.float64).cpu().numpy()))


@pytest.mark.parametrize("H,C", [(14, 1024), (7, 2048), (13, 256), (2, 8), (3, 16)])
def test_tap_bit_exact(H, C):
    A, A64 = bf(rng.standard_normal((3, H, H, C)))
    F = vista_tap(A).to(torch.float64).cpu().numpy()
    np.testing.assert_array_equal(F, oracle.tap(A64))


@pytest.mark.parametrize("H,k,s,C", [(114, 3, 2, 64), (55, 3, 2, 96), (13, 3, 2, 256), (224, 2, 2, 64), (7, 2, 2, 8)])
def test_maxpool_bit_exact(H, k, s, C):
    x, x64 = bf(rng.standard_normal((2, H, H, C)))
    np.testing.assert_array_equal(vista_maxpool(x, k, s).to(torch.float64).cpu().numpy(), oracle.maxpool(x64, k, s))


def test_avgpool():
    x, x64 = bf(rng.standard_normal((3, 7, 7, 2048)))
    got = vista_avgpool(x).to(torch.float64).cpu().numpy()
    assert normwise(got, oracle.avgpool_global(x64)) <= 4e-3


def test_lrn():
    x, x64 = bf(rng.standard_normal((2, 5, 5, 96)) * 20)
    got = vista_lrn(x).to(torch.float64).cpu().numpy()
    ref = oracle.lrn(x64)
    assert np.abs(got - ref).max() <= 4e-3 * np.abs(ref).max()


def test_ingest_exact():
    px = rng.integers(0, 256, (2, 227, 227, 3), dtype=np.uint8)
    y = vista_ingest(torch.from_numpy(px).cuda()).to(torch.float64).cpu().numpy()
    np.testing.assert_array_equal(y[..., :3], (px.astype(np.float64) - 128) / 128)
    assert not y[..., 3:].any()


@pytest.mark.parametrize("N", [24, 23])
def test_halo_cta_pair_bit_identical(monkeypatch, N):
    # the res3-class 3x3 halo conv runs as ONE tcgen05.mma.cta_group::2 per K step over both CTAs of a pair
    # (VISTA_CG2, default on) or as two cta_group::1 MMAs with multicast weights (VISTA_CG2=0): the same
    # per-element K order, so the same bits
    x, _ = bf(rng.standard_normal((N, 28, 28, 128)))
    w, _ = bf(rng.standard_normal((128, 3, 3, 128)) * (2.0 / 1152) ** 0.5)
    scale = torch.from_numpy(rng.uniform(0.5, 1.5, 128).astype(np.float32)).cuda()
    shift = torch.from_numpy(rng.standard_normal(128).astype(np.float32) * 0.1).cuda()
    out = {}
    for cg2 in ("1", "0"):
        monkeypatch.setenv("VISTA_CG2", cg2)
        out[cg2] = vista_conv2d(x, w, scale, shift, 1, 1, 1, relu=True).view(torch.int16).cpu()
    assert torch.equal(out["1"], out["0"])


@pytest.mark.parametrize("N,H,C,Cout,k,stride,residual", [
    (101, 14, 256, 256, 3, 1, False),   # res4 3x3 class: im2col A, odd M-tile count (phantom rank-1 tile)
    (200, 7, 512, 512, 3, 1, True),     # res5 3x3 class with a residual
    (100, 14, 1024, 256, 1, 1, False),  # 1x1 streamed weights: plain 2-D TMA A
    (100, 28, 512, 256, 1, 2, False),   # strided 1x1: im2col A with traversal stride 2, TMA epilogue
    (64, 7, 512, 2048, 1, 1, True),     # res5 closing conv: plain TMA A, 8 N tiles, TMA epilogue + residual
])
def test_pair_mma_bn256_bit_identical(monkeypatch, N, H, C, Cout, k, stride, residual):
    # BN = 256 im2col / plain-TMA convs run as ONE tcgen05.mma.cta_group::2 (M = 256, N = 256) per K step over the
    # multicast pair tile (VISTA_CG2 default on) or as two cta_group::1 MMAs with multicast weights (VISTA_CG2=0):
    # same per-element K order, same bits
    pad = (k - 1) // 2
    x, _ = bf(rng.standard_normal((N, H, H, C)))
    w, _ = bf(rng.standard_normal((Cout, k, k, C)) * (2.0 / (k * k * C)) ** 0.5)
    scale = torch.from_numpy(rng.uniform(0.5, 1.5, Cout).astype(np.float32)).cuda()
    shift = torch.from_numpy(rng.standard_normal(Cout).astype(np.float32) * 0.1).cuda()
    Ho = (H + 2 * pad - k) // stride + 1
    r = bf(rng.standard_normal((N, Ho, Ho, Cout)))[0] if residual else None
    out = {}
    for cg2 in ("1", "0"):
        monkeypatch.setenv("VISTA_CG2", cg2)
        out[cg2] = vista_conv2d(x, w, scale, shift, stride, pad, 1, residual=r, relu=True).view(torch.int16).cpu()
    assert torch.equal(out["1"], out["0"])


@pytest.mark.parametrize("N,H,C,Cout", [(13, 14, 256, 1024), (6, 28, 128, 512), (97, 14, 256, 1024)])
def test_a_multicast_bit_identical(monkeypatch, N, H, C, Cout):
    # resident-weight 1x1 convs with an even N-tile count run as CTA pairs that multicast each A k-block
    # (VISTA_AMC=1, opt-in: measured neutral): the same MMAs on the same operands as unicast A loads
    x, _ = bf(rng.standard_normal((N, H, H, C)))
    w, _ = bf(rng.standard_normal((Cout, 1, 1, C)) * (2.0 / C) ** 0.5)
    scale = torch.from_numpy(rng.uniform(0.5, 1.5, Cout).astype(np.float32)).cuda()
    shift = torch.from_numpy(rng.standard_normal(Cout).astype(np.float32) * 0.1).cuda()
    r = bf(rng.standard_normal((N, H, H, Cout)))[0]
    out = {}
    for amc in ("1", "0"):
        monkeypatch.setenv("VISTA_CG2_RES", "0")
        monkeypatch.setenv("VISTA_AMC", amc)
        out[amc] = vista_conv2d(x, w, scale, shift, 1, 0, 1, residual=r, relu=True).view(torch.int16).cpu()
    assert torch.equal(out["1"], out["0"])


@pytest.mark.parametrize("N,H,C,Cout", [(13, 14, 256, 1024), (6, 28, 128, 512), (97, 14, 256, 1024),
                                        (7, 56, 256, 64), (9, 56, 64, 64)])
def test_resident_weight_cta_pair_bit_identical(monkeypatch, N, H, C, Cout):
    # resident-weight 1x1 TMA-epilogue convs as CTA pairs (VISTA_CG2_RES, default on): two adjacent M tiles of
    # one N tile per pair, half of the N tile's weights per CTA, one M = 256 MMA per K step; odd M-tile counts
    # give rank 1 a phantom tile.  Same K order as one CTA per tile: same bits
    x, _ = bf(rng.standard_normal((N, H, H, C)))
    w, _ = bf(rng.standard_normal((Cout, 1, 1, C)) * (2.0 / C) ** 0.5)
    scale = torch.from_numpy(rng.uniform(0.5, 1.5, Cout).astype(np.float32)).cuda()
    shift = torch.from_numpy(rng.standard_normal(Cout).astype(np.float32) * 0.1).cuda()
    r = bf(rng.standard_normal((N, H, H, Cout)))[0]
    out = {}
    for flag in ("1", "0"):
        monkeypatch.setenv("VISTA_CG2_RES", flag)
        out[flag] = vista_conv2d(x, w, scale, shift, 1, 0, 1, residual=r, relu=True).view(torch.int16).cpu()
    assert torch.equal(out["1"], out["0"])


@pytest.mark.parametrize("N", [7, 24])
def test_halo64_cta_pair_bit_identical(monkeypatch, N):
    # res2-class 3x3 halo conv (Cout = 64, resident weights) as CTA pairs (VISTA_CG2_HALO64, default on): one
    # position in two consecutive images per pair tile, half of the resident weights per CTA, M = 256 MMAs; an
    # odd image count leaves rank 1 a phantom image.  Same K order as one CTA per tile: same bits
    x, _ = bf(rng.standard_normal((N, 56, 56, 64)))
    w, _ = bf(rng.standard_normal((64, 3, 3, 64)) * (2.0 / 576) ** 0.5)
    scale = torch.from_numpy(rng.uniform(0.5, 1.5, 64).astype(np.float32)).cuda()
    shift = torch.from_numpy(rng.standard_normal(64).astype(np.float32) * 0.1).cuda()
    out = {}
    for flag in ("1", "0"):
        monkeypatch.setenv("VISTA_CG2_HALO64", flag)
        out[flag] = vista_conv2d(x, w, scale, shift, 1, 1, 1, relu=True).view(torch.int16).cpu()
    assert torch.equal(out["1"], out["0"])


ROWCONV = [
    # N, H, W, relu   (3x3 / 1 / pad 1, Cin = Cout = 64: the input-row-major kernel, conv3x3_rows.cu)
    (2, 56, 56, True),     # res2 geometry, two bands
    (3, 56, 56, True),     # odd image count: phantom second image of the last pair
    (151, 56, 56, True),   # 152 items > 148 CTAs: CTAs own several (pair, band) items, TMEM ring wraps
    (1, 9, 11, False),     # small odd geometry, no ReLU, bands of 5 / 4 rows
    (5, 7, 62, True),      # widest supported row (62 + 2 padded columns = 64 A rows)
    (4, 1, 1, True),       # one row: only the centre filter row contributes
]


@pytest.mark.parametrize("N,H,W,relu", ROWCONV)
def test_rowconv3x3_bit_identical_to_halo(monkeypatch, N, H, W, relu):
    # the row kernel and the conv_tc halo / im2col path accumulate every output in the same (r, s, channel)
    # order, so they must agree bit for bit; both are checked against the oracle too
    x, x64 = bf(rng.standard_normal((N, H, W, 64)))
    w, w64 = bf(rng.standard_normal((64, 3, 3, 64)) * (2.0 / 576) ** 0.5)
    scale = rng.uniform(0.5, 1.5, 64).astype(np.float32)
    shift = rng.standard_normal(64).astype(np.float32) * 0.1
    out = {}
    for flag in ("1", "0"):
        monkeypatch.setenv("VISTA_ROWCONV", flag)
        out[flag] = vista_conv2d(x, w, torch.from_numpy(scale).cuda(), torch.from_numpy(shift).cuda(), 1, 1, 1,
                                 relu=relu)
        torch.cuda.synchronize()
    assert torch.equal(out["1"].view(torch.int16), out["0"].view(torch.int16))
    ref = oracle.conv2d(x64, w64, 1, 1, 1) * scale.astype(np.float64) + shift.astype(np.float64)
    if relu:
        ref = np.maximum(ref, 0)
    assert normwise(out["1"].to(torch.float64).cpu().numpy(), ref) <= 8e-3

"""ctypes wrapper of oracle/liboracle.so — the plain fp64 CPU oracle.

TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs may import this package.  The product path
(paper_conf_sigmod_nakandalak20_b200) never imports it and shares no code with it
except the seeded input generators in gen/.

Every function follows a passage of PAPER.md (cited in oracle/oracle.cpp); the
pins that tie it to something other than itself are in tests/test_oracle_*.py and
listed in DESIGN.md §"Oracle pins".
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

ALEXNET, VGG16, RESNET50 = 0, 1, 2
TAP_NAMES = {
    ALEXNET: ["conv5", "fc6", "fc7", "fc8"],
    VGG16: ["fc6", "fc7", "fc8"],
    RESNET50: ["conv4_6", "conv5_1", "conv5_2", "conv5_3", "fc"],
}

_vp = ctypes.c_void_p
_i64 = ctypes.c_int64


class LRCfg(ctypes.Structure):
    _fields_ = [("iters", ctypes.c_int32), ("power_iters", ctypes.c_int32),
                ("lam", ctypes.c_double), ("alpha", ctypes.c_double)]


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "liboracle.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `make oracle/liboracle.so` (or __graft_entry__.build())")
        L = ctypes.CDLL(path)
        i = ctypes.c_int
        L.or_conv2d.argtypes = [_vp, i, i, i, i, _vp, i, i, i, i, i, i, _vp, _vp]
        L.or_fc.argtypes = [_vp, i, i, _vp, i, _vp, _vp]
        L.or_maxpool.argtypes = [_vp, i, i, i, i, i, i, _vp]
        L.or_avgpool_global.argtypes = [_vp, i, i, i, i, _vp]
        L.or_lrn.argtypes = [_vp, i, i, i, i, _vp]
        L.or_batchnorm.argtypes = [_vp, _i64, i, _vp, _vp, _vp, _vp, ctypes.c_double, _vp]
        L.or_tap.argtypes = [_vp, i, i, i, i, _vp]
        L.oracle_cnn_info.argtypes = [i, i, _vp]
        L.oracle_features.argtypes = [i, ctypes.c_uint64, _vp, _i64, _vp, _vp, i]
        L.oracle_features_from.argtypes = [i, ctypes.c_uint64, i, _vp, _i64, _vp, _vp, i]
        L.oracle_join.argtypes = [_vp, _i64, _vp, _i64, ctypes.c_uint64, _vp, _vp, _vp, _vp]
        L.oracle_concat.argtypes = [_vp, i, _vp, i, _vp, _vp, _i64, _vp]
        L.oracle_lr_train.argtypes = [_vp, _i64, i, _vp, _vp, ctypes.POINTER(LRCfg), _vp, _vp, _vp, _vp, _vp]
        L.oracle_lr_stats.argtypes = [_vp, _i64, i, _vp, _vp, _vp, _vp]
        L.oracle_lr_objective.argtypes = [_vp, _i64, i, _vp, _vp, _vp, _vp, _vp, ctypes.c_double,
                                          ctypes.c_double, ctypes.c_double, _vp, _vp, _vp]
        L.oracle_lr_power.argtypes = [_vp, _i64, i, _vp, _vp, _vp, i, _vp]
        L.oracle_lr_grad_sums.argtypes = [_vp, _i64, i, _vp, _vp, _vp, ctypes.c_double, _vp]
        _LIB = L
    return _LIB


def _p(a):
    if a is None:
        return None
    assert a.flags["C_CONTIGUOUS"], "arrays passed to the oracle must be C-contiguous"
    return a.ctypes.data_as(_vp)


def _f64(a):
    return np.ascontiguousarray(a, dtype=np.float64)


def _chk(rc, what):
    if rc != 0:
        raise RuntimeError(f"oracle {what} failed with code {rc}")


# ---------------- primitives ----------------
def conv2d(x, w, stride=1, pad=0, groups=1, bias=None):
    """x NHWC, w OHWI [Cout, R, S, C/groups]."""
    x, w = _f64(x), _f64(w)
    N, H, W, C = x.shape
    Cout, R, S, _ = w.shape
    Ho, Wo = (H + 2 * pad - R) // stride + 1, (W + 2 * pad - S) // stride + 1
    y = np.empty((N, Ho, Wo, Cout))
    b = _f64(bias) if bias is not None else None
    _chk(lib().or_conv2d(_p(x), N, H, W, C, _p(w), Cout, R, S, stride, pad, groups, _p(b), _p(y)), "conv2d")
    return y


def fc(x, w, bias=None):
    x, w = _f64(x), _f64(w)
    N, K = x.shape
    y = np.empty((N, w.shape[0]))
    b = _f64(bias) if bias is not None else None
    _chk(lib().or_fc(_p(x), N, K, _p(w), w.shape[0], _p(b), _p(y)), "fc")
    return y


def maxpool(x, k, s):
    x = _f64(x)
    N, H, W, C = x.shape
    y = np.empty((N, (H - k) // s + 1, (W - k) // s + 1, C))
    _chk(lib().or_maxpool(_p(x), N, H, W, C, k, s, _p(y)), "maxpool")
    return y


def avgpool_global(x):
    x = _f64(x)
    N, H, W, C = x.shape
    y = np.empty((N, C))
    _chk(lib().or_avgpool_global(_p(x), N, H, W, C, _p(y)), "avgpool")
    return y


def lrn(x):
    x = _f64(x)
    N, H, W, C = x.shape
    y = np.empty_like(x)
    _chk(lib().or_lrn(_p(x), N, H, W, C, _p(y)), "lrn")
    return y


def batchnorm(x, gamma, beta, mean, var, eps=1e-5):
    x = _f64(x)
    C = x.shape[-1]
    y = np.empty_like(x)
    _chk(lib().or_batchnorm(_p(x), x.size // C, C, _p(_f64(gamma)), _p(_f64(beta)), _p(_f64(mean)),
                            _p(_f64(var)), eps, _p(y)), "batchnorm")
    return y


def tap(A):
    A = _f64(A)
    N, H, W, C = A.shape
    F = np.empty((N, 4 * C))
    _chk(lib().or_tap(_p(A), N, H, W, C, _p(F)), "tap")
    return F


# ---------------- roster / features ----------------
def cnn_info(cnn, t):
    out = np.zeros(8, dtype=np.int64)
    _chk(lib().oracle_cnn_info(cnn, t, _p(out)), "cnn_info")
    keys = ["H", "W", "C", "d", "macs", "macs_bias", "n_taps", "act"]
    return dict(zip(keys, (int(v) for v in out)))


def n_taps(cnn):
    return cnn_info(cnn, 0)["n_taps"]


def _ptr_array(arrs):
    a = (ctypes.c_void_p * len(arrs))()
    for i, x in enumerate(arrs):
        a[i] = x.ctypes.data if x is not None else None
    return a


def features(cnn, seed, images, taps, want_act=(), nthreads=0):
    """Eq. (2) for every tap in `taps` by a full fp64 forward from pixels.
    Returns ({tap: F [n, d]}, {tap: A [n, act]})."""
    images = np.ascontiguousarray(images, dtype=np.uint8)
    n = images.shape[0]
    T = n_taps(cnn)
    F = [None] * T
    A = [None] * T
    for t in taps:
        F[t] = np.empty((n, cnn_info(cnn, t)["d"]))
    for t in want_act:
        A[t] = np.empty((n, cnn_info(cnn, t)["act"]))
    _chk(lib().oracle_features(cnn, seed, _p(images), n, _ptr_array(F), _ptr_array(A), nthreads), "features")
    return ({t: F[t] for t in taps}, {t: A[t] for t in want_act})


def features_from(cnn, seed, t0, A_in, taps, want_act=(), nthreads=0):
    """Partial inference f^_{t0 -> t} (Def 3.7) from the stored activation of tap t0."""
    A_in = _f64(A_in)
    n = A_in.shape[0]
    T = n_taps(cnn)
    F = [None] * T
    A = [None] * T
    for t in taps:
        F[t] = np.empty((n, cnn_info(cnn, t)["d"]))
    for t in want_act:
        A[t] = np.empty((n, cnn_info(cnn, t)["act"]))
    _chk(lib().oracle_features_from(cnn, seed, t0, _p(A_in), n, _ptr_array(F), _ptr_array(A), nthreads),
         "features_from")
    return ({t: F[t] for t in taps}, {t: A[t] for t in want_act})


# ---------------- join / concat / LR ----------------
class DupKey(Exception):
    pass


def join(img_keys, str_keys, split_seed):
    img_keys = np.ascontiguousarray(img_keys, dtype=np.int64)
    str_keys = np.ascontiguousarray(str_keys, dtype=np.int64)
    ns = len(str_keys)
    ps = np.empty(max(ns, 1), dtype=np.int64)
    pi = np.empty(max(ns, 1), dtype=np.int64)
    te = np.empty(max(ns, 1), dtype=np.uint8)
    n = np.zeros(1, dtype=np.int64)
    rc = lib().oracle_join(_p(img_keys), len(img_keys), _p(str_keys), ns, split_seed, _p(ps), _p(pi), _p(te), _p(n))
    if rc == 3:
        raise DupKey("ID is not a primary key")
    _chk(rc, "join")
    k = int(n[0])
    return ps[:k].copy(), pi[:k].copy(), te[:k].copy()


def concat(X, F, pair_str, pair_img):
    X = np.ascontiguousarray(X, dtype=np.float32)
    F = _f64(F)
    ps = np.ascontiguousarray(pair_str, dtype=np.int64)
    pi = np.ascontiguousarray(pair_img, dtype=np.int64)
    d_s, d_l = X.shape[1], F.shape[1]
    MM = np.empty((len(ps), d_s + d_l))
    _chk(lib().oracle_concat(_p(X), d_s, _p(F), d_l, _p(ps), _p(pi), len(ps), _p(MM)), "concat")
    return MM


def lr_train(MM, y, is_test, iters=10, power_iters=20, lam=0.01, alpha=0.5):
    MM = _f64(MM)
    y = np.ascontiguousarray(y, dtype=np.uint8)
    te = np.ascontiguousarray(is_test, dtype=np.uint8)
    n, d = MM.shape
    cfg = LRCfg(iters, power_iters, lam, alpha)
    w = np.empty(d)
    b = np.zeros(1)
    loss = np.empty(max(iters, 1))
    lh = np.zeros(1)
    met = np.zeros(10)
    _chk(lib().oracle_lr_train(_p(MM), n, d, _p(y), _p(te), ctypes.byref(cfg), _p(w), _p(b), _p(loss), _p(lh),
                               _p(met)), "lr_train")
    names = ["train_acc", "test_acc", "test_f1", "n_train", "n_test", "tp", "fp", "tn", "fn", "eta"]
    return dict(w=w, b=float(b[0]), loss=loss[:iters], lambda_hat=float(lh[0]), **dict(zip(names, met.tolist())))


def lr_stats(MM, is_test):
    MM = _f64(MM)
    n, d = MM.shape
    te = np.ascontiguousarray(is_test, dtype=np.uint8) if is_test is not None else None
    mu, sig, inv = np.empty(d), np.empty(d), np.empty(d)
    _chk(lib().oracle_lr_stats(_p(MM), n, d, _p(te), _p(mu), _p(sig), _p(inv)), "lr_stats")
    return mu, sig, inv


def lr_objective(MM, y, is_test, mu, inv, w, b, lam, alpha):
    MM = _f64(MM)
    n, d = MM.shape
    te = np.ascontiguousarray(is_test, dtype=np.uint8) if is_test is not None else None
    f = np.zeros(1)
    gw = np.empty(d)
    gb = np.zeros(1)
    _chk(lib().oracle_lr_objective(_p(MM), n, d, _p(np.ascontiguousarray(y, dtype=np.uint8)), _p(te), _p(_f64(mu)),
                                   _p(_f64(inv)), _p(_f64(w)), float(b), lam, alpha, _p(f), _p(gw), _p(gb)),
         "lr_objective")
    return float(f[0]), gw, float(gb[0])


def lr_power(MM, is_test, mu, inv, K):
    MM = _f64(MM)
    n, d = MM.shape
    te = np.ascontiguousarray(is_test, dtype=np.uint8) if is_test is not None else None
    out = np.zeros(1)
    _chk(lib().oracle_lr_power(_p(MM), n, d, _p(te), _p(_f64(mu)), _p(_f64(inv)), K, _p(out)), "lr_power")
    return float(out[0])


def lr_grad_sums(MM, y, is_test, w_hat, b_hat):
    MM = _f64(MM)
    n, d = MM.shape
    te = np.ascontiguousarray(is_test, dtype=np.uint8) if is_test is not None else None
    out = np.empty(d + 2)
    _chk(lib().oracle_lr_grad_sums(_p(MM), n, d, _p(np.ascontiguousarray(y, dtype=np.uint8)), _p(te),
                                   _p(_f64(w_hat)), float(b_hat), _p(out)), "lr_grad_sums")
    return out

"""Seeded synthetic-input generators (ctypes wrapper of gen/libvista_gen.so).

Shared by the tests, bench.py, the CPU oracle and the CUDA path.  Holds no method
arithmetic: only counter-based random numbers and the data recipe of DESIGN.md
§"Input recipe" (SURVEY.md §8d "Generator").  Paper context: T_str(ID, X),
T_img(ID, I) (§3.2), Foods/Amazon shapes.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

DEFAULT_SEED = 0x5EED2020
IMG_H = IMG_W = 227
IMG_C = 3
IMG_BYTES = IMG_H * IMG_W * IMG_C
FOODS, AMAZON = 0, 1

_i64p = ctypes.POINTER(ctypes.c_int64)


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libvista_gen.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `make gen/libvista_gen.so` (or __graft_entry__.build())")
        L = ctypes.CDLL(path)
        L.vg_mix64.restype = ctypes.c_uint64
        L.vg_mix64.argtypes = [ctypes.c_uint64]
        L.vg_subseed.restype = ctypes.c_uint64
        L.vg_subseed.argtypes = [ctypes.c_uint64, ctypes.c_uint64]
        L.vg_latent.restype = ctypes.c_int
        L.vg_latent.argtypes = [ctypes.c_uint64, ctypes.c_int64]
        L.vg_keys.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_int64, ctypes.c_void_p]
        L.vg_images.argtypes = [ctypes.c_uint64, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p]
        L.vg_structured.argtypes = [ctypes.c_uint64, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32,
                                    ctypes.c_int32, ctypes.c_void_p]
        L.vg_labels.argtypes = [ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64,
                                ctypes.c_int32, ctypes.c_void_p]
        L.vg_str_rows.restype = ctypes.c_int64
        L.vg_str_rows.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_int32, ctypes.c_void_p]
        L.vg_param.argtypes = [ctypes.c_uint64, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, ctypes.c_int64,
                               ctypes.c_int32, ctypes.c_double, ctypes.c_double, ctypes.c_int32, ctypes.c_void_p]
        L.vg_bf16_round.restype = ctypes.c_float
        L.vg_bf16_round.argtypes = [ctypes.c_double]
        L.vg_set_threads.argtypes = [ctypes.c_int]
        _LIB = L
    return _LIB


def _p(a: np.ndarray):
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(ctypes.c_void_p)


def mix64(x: int) -> int:
    return lib().vg_mix64(x & 0xFFFFFFFFFFFFFFFF)


def subseed(S: int, k: int) -> int:
    return lib().vg_subseed(S & 0xFFFFFFFFFFFFFFFF, k)


def keys(seed: int, r0: int, n: int) -> np.ndarray:
    out = np.empty(n, dtype=np.int64)
    if n:
        lib().vg_keys(seed, r0, n, _p(out))
    return out


def keys_for_rows(seed: int, rows: np.ndarray) -> np.ndarray:
    # key_r = mix64(S_key + r); computed through the C generator one contiguous run at a time
    out = np.empty(len(rows), dtype=np.int64)
    full = keys(seed, 0, int(rows.max()) + 1) if len(rows) else out
    out[:] = full[rows]
    return out


def latent(seed: int, key: int) -> int:
    return lib().vg_latent(seed, int(key))


def images(seed: int, img_keys: np.ndarray, out: np.ndarray | None = None) -> np.ndarray:
    img_keys = np.ascontiguousarray(img_keys, dtype=np.int64)
    n = len(img_keys)
    if out is None:
        out = np.empty((n, IMG_H, IMG_W, IMG_C), dtype=np.uint8)
    assert out.dtype == np.uint8 and out.size == n * IMG_BYTES and out.flags["C_CONTIGUOUS"]
    if n:
        lib().vg_images(seed, _p(img_keys), n, out.ctypes.data_as(ctypes.c_void_p))
    return out


def structured(seed: int, k: np.ndarray, d_s: int, kind: int) -> np.ndarray:
    k = np.ascontiguousarray(k, dtype=np.int64)
    out = np.empty((len(k), d_s), dtype=np.float32)
    if len(k) and d_s:
        lib().vg_structured(seed, _p(k), len(k), d_s, kind, _p(out))
    return out


def labels(seed: int, k: np.ndarray, X: np.ndarray) -> np.ndarray:
    k = np.ascontiguousarray(k, dtype=np.int64)
    X = np.ascontiguousarray(X, dtype=np.float32)
    out = np.empty(len(k), dtype=np.uint8)
    if len(k):
        lib().vg_labels(seed, _p(k), _p(X), len(k), X.shape[1], _p(out))
    return out


def str_rows(seed: int, N: int, mismatch: bool) -> np.ndarray:
    buf = np.empty(N + N // 100 + 1, dtype=np.int64)
    n = lib().vg_str_rows(seed, N, 1 if mismatch else 0, _p(buf))
    return buf[:n].copy()


def param(seed: int, cnn: int, layer: int, tensor: int, n: int, kind: int, mean: float, std: float,
          round_bf16: bool) -> np.ndarray:
    out = np.empty(n, dtype=np.float64)
    if n:
        lib().vg_param(seed, cnn, layer, tensor, n, kind, mean, std, 1 if round_bf16 else 0, _p(out))
    return out


def set_threads(n: int) -> None:
    lib().vg_set_threads(int(n))


@dataclass
class Tables:
    """T_img(ID, I) for image rows [r0, r0+n_img) and the whole T_str(ID, X) + labels."""
    img_keys: np.ndarray      # int64 [n_img]
    images: np.ndarray | None  # uint8 [n_img, 227, 227, 3]
    str_keys: np.ndarray      # int64 [n_str]
    X: np.ndarray             # float32 [n_str, d_s]
    labels: np.ndarray        # uint8 [n_str]


def make_tables(N: int, d_s: int, kind: int = FOODS, seed: int = DEFAULT_SEED, mismatch: bool = False,
                r0: int = 0, n_img: int | None = None, with_images: bool = True) -> Tables:
    """Image rows r0 .. r0+n_img (a rank's contiguous shard) of an N-row image table,
    plus the full structured table (replicated on every rank: the broadcast join of
    PAPER.md:279)."""
    if n_img is None:
        n_img = N - r0
    img_keys = keys(seed, r0, n_img)
    rows = str_rows(seed, N, mismatch)
    all_keys = keys(seed, 0, N + N // 100 + 1)
    str_keys = np.ascontiguousarray(all_keys[rows])
    X = structured(seed, str_keys, d_s, kind)
    y = labels(seed, str_keys, X)
    imgs = images(seed, img_keys) if with_images else None
    return Tables(img_keys, imgs, str_keys, X, y)

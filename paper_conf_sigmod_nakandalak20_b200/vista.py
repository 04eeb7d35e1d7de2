"""Thin ctypes binding of libvista.so (include/vista.h).

Argument marshalling only: every step of the path runs in the library's sm_100a
kernels.  torch is used for device memory and streams; numpy arrays are host inputs.
There is no CPU fallback: if the extension is missing or no sm_100 GPU is present,
every call raises.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# VISTA_LIB_PATH: another build of the same library (A/B measurements of two builds in one job only)
LIB_PATH = os.environ.get("VISTA_LIB_PATH") or os.path.join(_HERE, "libvista.so")
_LIB = None

ALEXNET, VGG16, RESNET50 = 0, 1, 2
TAP_NAMES = {ALEXNET: ["conv5", "fc6", "fc7", "fc8"], VGG16: ["fc6", "fc7", "fc8"],
             RESNET50: ["conv4_6", "conv5_1", "conv5_2", "conv5_3", "fc"]}
STATUS = {0: "ok", 1: "invalid argument", 2: "no plan", 3: "duplicate key", 4: "state", 5: "cuda", 6: "nccl", 7: "oom"}

_vp = ctypes.c_void_p
_i32, _i64, _u64, _f64 = ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64, ctypes.c_double


class VistaError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"vista error {status} ({STATUS.get(status, '?')}): {msg}")
        self.status = status


class LRCfg(ctypes.Structure):
    _fields_ = [("iters", _i32), ("power_iters", _i32), ("lam", _f64), ("alpha", _f64), ("split_seed", _u64)]


# int32_t (*allreduce)(void* host_buf, int64_t count, int32_t dtype, void* user) of vista_sys_cfg
ALLREDUCE_FN = ctypes.CFUNCTYPE(_i32, _vp, _i64, _i32, _vp)


class SysCfg(ctypes.Structure):
    _fields_ = [("rank", _i32), ("world", _i32), ("nccl_uid", _vp), ("device", _i32), ("hbm_budget_bytes", _u64),
                ("dtype", _i32), ("plan", _i32), ("stream", _vp), ("micro_batch", _i32),
                ("allreduce", ALLREDUCE_FN), ("allreduce_user", _vp)]


class PlanInfo(ctypes.Structure):
    _fields_ = [("n_layers", _i32), ("tap", _i32 * 8), ("d_l", _i32 * 8), ("ld", _i32 * 8),
                ("micro_batch", _i32 * 8), ("act_bytes", _i64 * 8), ("peak_bytes_pred", _i64),
                ("weight_bytes", _i64), ("d_s", _i32), ("ds_pad", _i32), ("chunk_images", _i64),
                ("peak_bytes_meas", _i64), ("peak_reserved_meas", _i64), ("cnn_graph", _i32),
                ("cnn_graph_kernels", _i32)]


class Buffer(ctypes.Structure):
    _fields_ = [("mm", _vp), ("rows", _i64), ("n_train", _i64), ("ld", _i32), ("d_s", _i32), ("ds_pad", _i32),
                ("d_l", _i32), ("pair_str", _vp), ("pair_img", _vp), ("labels", _vp), ("features", _vp),
                ("activation", _vp)]


class Metrics(ctypes.Structure):
    _fields_ = [("loss", _f64 * 64), ("lambda_hat", _f64), ("eta", _f64), ("train_acc", _f64), ("test_acc", _f64),
                ("test_f1", _f64), ("n_train", _i64), ("n_test", _i64), ("tp", _i64), ("fp", _i64), ("tn", _i64),
                ("fn", _i64)]


class Profile(ctypes.Structure):
    _fields_ = [("ms", _f64 * 8), ("launches", _i64 * 8), ("flops", _f64 * 8), ("bytes", _f64 * 8),
                ("roof_ms", _f64 * 8)]


PROFILE_CLASSES = ["conv_fc_tcgen05", "tap", "pool_cvt_lrn", "join", "concat", "lr_pass", "lr_small", "mlp"]


class MLPCfg(ctypes.Structure):
    _fields_ = [("hidden", _i32), ("iters", _i32), ("lr", _f64), ("seed", _u64)]


def lib():
    global _LIB
    if _LIB is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: build it with `make` or __graft_entry__.build() "
                               "(there is no CPU fallback)")
        L = ctypes.CDLL(LIB_PATH)
        L.vista_status_str.restype = ctypes.c_char_p
        L.vista_last_error.restype = ctypes.c_char_p
        L.vista_last_error.argtypes = [_vp]
        L.vista_plan.argtypes = [_i32, _vp, _i32, _i32, _i64, _i32, _i64, ctypes.POINTER(LRCfg),
                                 ctypes.POINTER(SysCfg), _u64, ctypes.POINTER(_vp)]
        L.vista_plan_info.argtypes = [_vp, ctypes.POINTER(PlanInfo)]
        L.vista_transfer.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp]
        L.vista_features.argtypes = [_vp, _i32, ctypes.POINTER(Buffer)]
        L.vista_train_mlp.argtypes = [_vp, _i32, ctypes.POINTER(MLPCfg), _vp, ctypes.POINTER(Metrics)]
        L.vista_base_shape.argtypes = [_vp, ctypes.POINTER(_i64)]
        L.vista_materialize.argtypes = [_vp, _vp, _vp]
        L.vista_transfer_from_base.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp]
        L.vista_train.argtypes = [_vp, _i32, _vp, ctypes.POINTER(Metrics)]
        L.vista_run.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp, _vp, _vp]
        L.vista_destroy.argtypes = [_vp]
        L.vista_destroy.restype = None
        L.vista_shard_range.argtypes = [_i64, _i32, _i32, ctypes.POINTER(_i64), ctypes.POINTER(_i64)]
        L.vista_shard_range.restype = None
        L.vista_nccl_unique_id.argtypes = [_vp]
        L.vista_set_profiling.argtypes = [_vp, _i32]
        L.vista_get_profile.argtypes = [_vp, ctypes.POINTER(Profile), _i32]
        L.vista_set_roofline.argtypes = [_vp, _f64, _f64]
        L.vista_conv2d.argtypes = [_vp, _i32, _i32, _i32, _i32, _vp, _i32, _i32, _i32, _i32, _i32, _i32, _vp, _vp,
                                   _vp, _i32, _vp, _vp]
        L.vista_conv2d_tap.argtypes = [_vp, _i32, _i32, _i32, _i32, _vp, _i32, _i32, _i32, _i32, _i32, _vp, _vp,
                                       _vp, _vp, _vp, _vp]
        L.vista_kernel_launches.restype = _i64
        L.vista_tap.argtypes = [_vp, _i32, _i32, _i32, _i32, _vp, _vp]
        L.vista_join.argtypes = [_vp, _i64, _vp, _i64, _u64, _vp, _vp, ctypes.POINTER(_i64), ctypes.POINTER(_i64),
                                 _vp]
        L.vista_maxpool.argtypes = [_vp, _i32, _i32, _i32, _i32, _i32, _i32, _vp, _vp]
        L.vista_lrn.argtypes = [_vp, _i32, _i32, _i32, _i32, _vp, _vp]
        L.vista_avgpool.argtypes = [_vp, _i32, _i32, _i32, _i32, _vp, _vp]
        L.vista_ingest.argtypes = [_vp, _i32, _vp, _vp]
        _LIB = L
    return _LIB


def _check(rc, ctx=None):
    if rc != 0:
        msg = lib().vista_last_error(ctx)
        raise VistaError(rc, msg.decode() if msg else "")


def _ptr(a):
    """Data pointer of a numpy array (host) or torch tensor (host or device)."""
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        assert a.flags["C_CONTIGUOUS"]
        return a.ctypes.data
    assert a.is_contiguous()
    return a.data_ptr()


def _stream(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    return stream


# ---------------- C-ABI mirrors ----------------
def vista_shard_range(n, rank, world):
    b, e = _i64(), _i64()
    lib().vista_shard_range(n, rank, world, ctypes.byref(b), ctypes.byref(e))
    return b.value, e.value


def vista_nccl_unique_id() -> bytes:
    buf = (ctypes.c_uint8 * 128)()
    _check(lib().vista_nccl_unique_id(buf))
    return bytes(buf)


def vista_conv2d(x, w, scale, shift, stride=1, pad=0, groups=1, residual=None, relu=False, y=None, stream=None):
    """x bf16 NHWC cuda tensor, w bf16 OHWI; returns y bf16 NHWC."""
    import torch
    N, H, W, C = x.shape
    Cout, R, S, _ = w.shape
    Ho, Wo = (H + 2 * pad - R) // stride + 1, (W + 2 * pad - S) // stride + 1
    if y is None:
        y = torch.empty((N, Ho, Wo, Cout), dtype=torch.bfloat16, device=x.device)
    _check(lib().vista_conv2d(_ptr(x), N, H, W, C, _ptr(w), Cout, R, S, stride, pad, groups, _ptr(scale),
                              _ptr(shift), _ptr(residual), 1 if relu else 0, _ptr(y), _stream(stream)))
    return y


def vista_conv2d_tap(x, w, scale, shift, stride=1, pad=0, residual=None, stream=None):
    """conv + ReLU with the 2x2-grid tap fused into the epilogue; returns (y, F)."""
    import torch
    N, H, W, C = x.shape
    Cout, R, S, _ = w.shape
    Ho, Wo = (H + 2 * pad - R) // stride + 1, (W + 2 * pad - S) // stride + 1
    y = torch.empty((N, Ho, Wo, Cout), dtype=torch.bfloat16, device=x.device)
    F = torch.empty((N, 4 * Cout), dtype=torch.bfloat16, device=x.device)
    _check(lib().vista_conv2d_tap(_ptr(x), N, H, W, C, _ptr(w), Cout, R, S, stride, pad, _ptr(scale), _ptr(shift),
                                  _ptr(residual), _ptr(y), _ptr(F), _stream(stream)))
    return y, F


def vista_join(img_keys, str_keys, split_seed=0, stream=None):
    """S4 join on its own: device int64 key tensors -> (pair_str, pair_img) int32 device tensors of the
    matched rows ([train | test], each in T_str order) and n_train."""
    import torch
    ns = str_keys.shape[0]
    ps = torch.empty(max(ns, 1), dtype=torch.int32, device=str_keys.device)
    pi = torch.empty(max(ns, 1), dtype=torch.int32, device=str_keys.device)
    n_pairs, n_train = _i64(), _i64()
    _check(lib().vista_join(_ptr(img_keys), img_keys.shape[0], _ptr(str_keys), ns, split_seed, _ptr(ps), _ptr(pi),
                            ctypes.byref(n_pairs), ctypes.byref(n_train), _stream(stream)))
    return ps[:n_pairs.value], pi[:n_pairs.value], n_train.value


def torch_dist_allreduce(group=None):
    """An allreduce for vista_sys_cfg.allreduce backed by a torch.distributed process group (e.g. gloo):
    in-place SUM of the library's host buffer.  Marshalling only (the sums the library asks for are its
    own per-rank partials)."""
    import torch
    import torch.distributed as dist

    def fn(buf, count, dtype, user):
        try:
            ct = ctypes.c_double if dtype == 0 else ctypes.c_float
            arr = np.ctypeslib.as_array((ct * count).from_address(buf))
            t = torch.from_numpy(arr)
            dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
            return 0
        except Exception:  # never raise through the C frame
            return 1
    return fn


def vista_kernel_launches() -> int:
    return int(lib().vista_kernel_launches())


def vista_tap(A, stream=None):
    import torch
    N, H, W, C = A.shape
    F = torch.empty((N, 4 * C), dtype=torch.bfloat16, device=A.device)
    _check(lib().vista_tap(_ptr(A), N, H, W, C, _ptr(F), _stream(stream)))
    return F


def vista_maxpool(x, k, s, stream=None):
    import torch
    N, H, W, C = x.shape
    y = torch.empty((N, (H - k) // s + 1, (W - k) // s + 1, C), dtype=torch.bfloat16, device=x.device)
    _check(lib().vista_maxpool(_ptr(x), N, H, W, C, k, s, _ptr(y), _stream(stream)))
    return y


def vista_lrn(x, stream=None):
    import torch
    y = torch.empty_like(x)
    N, H, W, C = x.shape
    _check(lib().vista_lrn(_ptr(x), N, H, W, C, _ptr(y), _stream(stream)))
    return y


def vista_avgpool(x, stream=None):
    import torch
    N, H, W, C = x.shape
    y = torch.empty((N, C), dtype=torch.bfloat16, device=x.device)
    _check(lib().vista_avgpool(_ptr(x), N, H, W, C, _ptr(y), _stream(stream)))
    return y


def vista_ingest(px, stream=None):
    import torch
    N = px.shape[0]
    y = torch.empty((N, 227, 227, 8), dtype=torch.bfloat16, device=px.device)
    _check(lib().vista_ingest(_ptr(px), N, _ptr(y), _stream(stream)))
    return y


class _CudaView:
    """Zero-copy view of library-owned device memory for torch.as_tensor."""

    def __init__(self, ptr, shape, typestr):
        self.__cuda_array_interface__ = {"shape": tuple(int(s) for s in shape), "typestr": typestr,
                                         "data": (int(ptr or 0), False), "version": 3, "strides": None}


def _dev_tensor(ptr, shape, typestr, dtype=None):
    import torch
    n = int(np.prod(shape))
    if n == 0 or not ptr:
        t = torch.empty(shape, dtype={"<i2": torch.int16, "<f4": torch.float32, "<i4": torch.int32,
                                      "|u1": torch.uint8}.get(typestr), device="cuda")
    else:
        t = torch.as_tensor(_CudaView(ptr, shape, typestr), device="cuda")
    return t.view(dtype) if dtype is not None else t


class Vista:
    """One ctx: vista_plan -> vista_transfer -> vista_train(k)."""

    def __init__(self, cnn, layers=None, n_top=0, n_str_rows=0, d_s=0, n_images_local=0, iters=10,
                 power_iters=20, lam=0.01, alpha=0.5, split_seed=0, weight_seed=0, rank=0, world=1,
                 nccl_uid: bytes | None = None, device=0, hbm_budget_bytes=0, stream=None, micro_batch=0,
                 plan="staged", dtype="bf16", allreduce=None):
        """dtype: "bf16" (the tcgen05 product path) or "f32" (the fp32 check mode, reading R23).
        allreduce: a Python callable fn(host_ptr, count, dtype, user) -> int (e.g. torch_dist_allreduce())
        used instead of NCCL when world > 1 and nccl_uid is None."""
        self.cnn = cnn
        self.dtype = dtype
        lr = LRCfg(iters, power_iters, lam, alpha, split_seed)
        self._uid = (ctypes.c_uint8 * 128).from_buffer_copy(nccl_uid) if nccl_uid else None
        plan_id = {"staged": 0, "eager": 1, "lazy": 2}[plan]
        dtype_id = {"bf16": 0, "f32": 1}[dtype]
        self._ar = ALLREDUCE_FN(allreduce) if allreduce is not None else ALLREDUCE_FN()  # kept alive with self
        sys = SysCfg(rank, world, ctypes.addressof(self._uid) if self._uid is not None else None, device,
                     hbm_budget_bytes, dtype_id, plan_id, stream, micro_batch, self._ar, None)
        arr = None
        n_layers = 0
        if layers is not None:
            arr = (_i32 * len(layers))(*layers)
            n_layers = len(layers)
        ctx = _vp()
        rc = lib().vista_plan(cnn, arr, n_layers, n_top, n_str_rows, d_s, n_images_local, ctypes.byref(lr),
                              ctypes.byref(sys), weight_seed, ctypes.byref(ctx))
        _check(rc, None)
        self.ctx = ctx
        self.n_images_local = n_images_local

    def plan_info(self):
        pi = PlanInfo()
        _check(lib().vista_plan_info(self.ctx, ctypes.byref(pi)), self.ctx)
        n = pi.n_layers
        return dict(n_layers=n, tap=list(pi.tap[:n]), d_l=list(pi.d_l[:n]), ld=list(pi.ld[:n]),
                    micro_batch=list(pi.micro_batch[:n]), act_bytes=list(pi.act_bytes[:n]),
                    peak_bytes_pred=pi.peak_bytes_pred, weight_bytes=pi.weight_bytes, d_s=pi.d_s, ds_pad=pi.ds_pad,
                    chunk_images=pi.chunk_images, peak_bytes_meas=pi.peak_bytes_meas,
                    peak_reserved_meas=pi.peak_reserved_meas, cnn_graph=pi.cnn_graph,
                    cnn_graph_kernels=pi.cnn_graph_kernels)

    def transfer(self, images, image_keys, structured, str_keys, labels):
        _check(lib().vista_transfer(self.ctx, _ptr(images), _ptr(image_keys), _ptr(structured), _ptr(str_keys),
                                    _ptr(labels)), self.ctx)

    def base_shape(self):
        """(H, W, C, bytes per element) of one image's base-layer activation A_{L[0]} (App. B)."""
        o = (_i64 * 4)()
        _check(lib().vista_base_shape(self.ctx, o), self.ctx)
        return tuple(int(v) for v in o)

    def materialize(self, images, base_out):
        """base_out <- A_{L[0]} of every local image (NHWC, host or device tensor / array)."""
        _check(lib().vista_materialize(self.ctx, _ptr(images), _ptr(base_out)), self.ctx)

    def transfer_from_base(self, base, image_keys, structured, str_keys, labels):
        """vista_transfer started at the pre-materialised base layer (App. B)."""
        _check(lib().vista_transfer_from_base(self.ctx, _ptr(base), _ptr(image_keys), _ptr(structured),
                                              _ptr(str_keys), _ptr(labels)), self.ctx)

    def features(self, k):
        import torch
        b = Buffer()
        _check(lib().vista_features(self.ctx, k, ctypes.byref(b)), self.ctx)
        rows = b.rows
        ts, tdt = ("<f4", None) if self.dtype == "f32" else ("<i2", torch.bfloat16)
        return dict(
            mm=_dev_tensor(b.mm, (rows, b.ld), ts, tdt),
            rows=rows, n_train=b.n_train, ld=b.ld, d_s=b.d_s, ds_pad=b.ds_pad, d_l=b.d_l,
            pair_str=_dev_tensor(b.pair_str, (rows,), "<i4"),
            pair_img=_dev_tensor(b.pair_img, (rows,), "<i4"),
            labels=_dev_tensor(b.labels, (rows,), "|u1"),
            features=_dev_tensor(b.features, (self.n_images_local, b.d_l), ts, tdt),
            has_activation=bool(b.activation),
        )

    def train(self, k, d_total):
        w = np.zeros(d_total + 1, dtype=np.float64)
        m = Metrics()
        _check(lib().vista_train(self.ctx, k, w.ctypes.data, ctypes.byref(m)), self.ctx)
        T = 64
        met = dict(loss=list(m.loss[:T]), lambda_hat=m.lambda_hat, eta=m.eta, train_acc=m.train_acc,
                   test_acc=m.test_acc, test_f1=m.test_f1, n_train=m.n_train, n_test=m.n_test, tp=m.tp, fp=m.fp,
                   tn=m.tn, fn=m.fn)
        return w[:-1], float(w[-1]), met

    def run(self, images, image_keys, structured, str_keys, labels, d_totals, want_weights=True):
        """vista_run: transfer + M of every layer (M(k) beside stage k+1; VISTA_LR_BATCH=1: side by side after the
        transfer); returns [(w, b, metrics)] per layer."""
        L = len(d_totals)
        ws = [np.zeros(d + 1, dtype=np.float64) for d in d_totals] if want_weights else None
        ptrs = (ctypes.c_void_p * L)(*[w.ctypes.data for w in ws]) if want_weights else None
        ms = (Metrics * L)()
        _check(lib().vista_run(self.ctx, _ptr(images), _ptr(image_keys), _ptr(structured), _ptr(str_keys),
                               _ptr(labels), ptrs, ms), self.ctx)
        out = []
        for k in range(L):
            m = ms[k]
            met = dict(loss=list(m.loss[:64]), lambda_hat=m.lambda_hat, eta=m.eta, train_acc=m.train_acc,
                       test_acc=m.test_acc, test_f1=m.test_f1, n_train=m.n_train, n_test=m.n_test, tp=m.tp,
                       fp=m.fp, tn=m.tn, fn=m.fn)
            out.append((ws[k][:-1], float(ws[k][-1]), met) if want_weights else (None, None, met))
        return out

    def train_mlp(self, k, d_total, iters=10, lr=0.01, seed=0, hidden=1024, want_weights=True):
        """3-layer MLP (reading R30) on layer k; returns (params dict or None, metrics)."""
        h, d = hidden, d_total
        w = np.zeros(h * d + h + h * h + h + h + 1, dtype=np.float32) if want_weights else None
        m = Metrics()
        cfg = MLPCfg(hidden, iters, lr, seed)
        _check(lib().vista_train_mlp(self.ctx, k, ctypes.byref(cfg), w.ctypes.data if want_weights else None,
                                     ctypes.byref(m)), self.ctx)
        met = dict(loss=list(m.loss[:iters]), train_acc=m.train_acc, test_acc=m.test_acc, test_f1=m.test_f1,
                   n_train=m.n_train, n_test=m.n_test, tp=m.tp, fp=m.fp, tn=m.tn, fn=m.fn, lr=m.eta)
        if not want_weights:
            return None, met
        o = 0
        P = {}
        for name, shape in (("W1", (h, d)), ("b1", (h,)), ("W2", (h, h)), ("b2", (h,)), ("w3", (h,))):
            size = int(np.prod(shape))
            P[name] = w[o:o + size].reshape(shape).astype(np.float64)
            o += size
        P["b3"] = float(w[o])
        return P, met

    def set_profiling(self, on: bool):
        _check(lib().vista_set_profiling(self.ctx, 1 if on else 0), self.ctx)

    def profile(self, reset=True):
        p = Profile()
        _check(lib().vista_get_profile(self.ctx, ctypes.byref(p), 1 if reset else 0), self.ctx)
        return {name: dict(ms=p.ms[i], launches=p.launches[i], flops=p.flops[i], bytes=p.bytes[i],
                           roof_ms=p.roof_ms[i])
                for i, name in enumerate(PROFILE_CLASSES)}

    def set_roofline(self, tflops, gbps):
        _check(lib().vista_set_roofline(self.ctx, float(tflops), float(gbps)), self.ctx)

    def close(self):
        if getattr(self, "ctx", None):
            lib().vista_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

"""B200-native KDE range-selectivity hot path (Heimel, Kiefer, Markl, SIGMOD 2015).

Thin ctypes binding over the C ABI of ``include/kde.h`` (``libkde.so``, built
in-tree for sm_100a by ``build.py``).  This module only marshals arguments:
every numeric step runs in the library's CUDA kernels.  There is no CPU
fallback -- if ``libkde.so`` is missing or no CUDA device is present the calls
fail loudly.

Function names mirror the C ABI (``kde_create``, ``kde_estimate_batch``,
``kde_loss_and_grad``, ``kde_karma_update``, ``kde_replace_points``, ...);
``KDEModel`` is a small convenience wrapper that owns the handle.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("KDE_LIB_PATH") or os.path.join(_HERE, "libkde.so")  # override: tuning builds

KDE_OK, KDE_EINVAL, KDE_ENOMEM, KDE_ECUDA, KDE_ENCCL, KDE_ESTATE, KDE_ETRUNC = range(7)
LOSS_SQUARED, LOSS_ABSOLUTE, LOSS_RELATIVE, LOSS_SQUARED_RELATIVE, LOSS_SQUARED_Q = range(5)
KERNEL_GAUSSIAN, KERNEL_EPANECHNIKOV = 0, 1
KDE_MAX_DIM = 16
KDE_NCCL_ID_BYTES = 128
KDE_PEER_HANDLE_BYTES = 64

# every symbol include/kde.h declares (checked by tests/test_abi.py)
ABI_SYMBOLS = (
    "kde_abi_version", "kde_last_error", "kde_status_string", "kde_create", "kde_create_sharded",
    "kde_get_unique_id", "kde_destroy", "kde_get_info", "kde_get_bandwidth", "kde_set_bandwidth",
    "kde_set_retain", "kde_estimate_batch", "kde_estimate_batch_dev", "kde_loss_and_grad",
    "kde_loss_and_grad_dev", "kde_karma_update", "kde_online_update", "kde_replace_points",
    "kde_get_karma", "kde_set_karma", "kde_get_sample", "kde_get_contributions", "kde_get_online_state",
    "kde_set_online_state", "kde_synchronize", "kde_count_in_box_dev", "kde_set_profiling", "kde_get_profile",
    "kde_karma_update_dev", "kde_online_update_dev", "kde_replace_points_dev", "kde_stream_step_dev",
    "kde_set_kernel", "kde_get_kernel", "kde_set_cull", "kde_get_cull", "kde_set_cells", "kde_get_cells",
    "kde_reservoir_select", "kde_insert_rows", "kde_insert_rows_async",
    "kde_create_sharded_peer", "kde_peer_handle", "kde_peer_attach",
)


class KDEError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


_STATUS = {0: "KDE_OK", 1: "KDE_EINVAL", 2: "KDE_ENOMEM", 3: "KDE_ECUDA", 4: "KDE_ENCCL", 5: "KDE_ESTATE",
           6: "KDE_ETRUNC"}


class KarmaParams(ctypes.Structure):
    """kde_karma_params (include/kde.h): eq. (7)-(8)."""
    _fields_ = [("loss", ctypes.c_int32), ("empty_region", ctypes.c_int32), ("lambda_", ctypes.c_double),
                ("k_max", ctypes.c_double), ("k_init", ctypes.c_double), ("threshold", ctypes.c_double)]


class OnlineParams(ctypes.Structure):
    """kde_online_params (include/kde.h): Listing 1 knobs, defaults of P:L183."""
    _fields_ = [("minibatch", ctypes.c_int32), ("log_bandwidth", ctypes.c_int32), ("loss", ctypes.c_int32),
                ("_pad", ctypes.c_int32), ("lambda_", ctypes.c_double), ("alpha", ctypes.c_double),
                ("lr_min", ctypes.c_double), ("lr_max", ctypes.c_double), ("lr_inc", ctypes.c_double),
                ("lr_dec", ctypes.c_double), ("lr0", ctypes.c_double)]


def karma_params(loss=LOSS_ABSOLUTE, lam=0.0, k_max=4.0, k_init=0.0, threshold=0.0, empty_region=True):
    return KarmaParams(loss, int(bool(empty_region)), lam, k_max, k_init, threshold)


def online_params(minibatch=10, log_bandwidth=True, loss=LOSS_ABSOLUTE, lam=0.0, alpha=0.9, lr_min=1e-6,
                  lr_max=50.0, lr_inc=1.2, lr_dec=0.5, lr0=0.1):
    return OnlineParams(minibatch, int(bool(log_bandwidth)), loss, 0, lam, alpha, lr_min, lr_max, lr_inc, lr_dec,
                        lr0)


_lib = None


def lib() -> ctypes.CDLL:
    """Load libkde.so (raises if it was not built -- there is no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not found: build it with `python -m paper_conf_sigmod_heimelkm15_b200.build` "
                          "(there is no CPU fallback)")
    L = ctypes.CDLL(LIB_PATH)
    P, i32, i64, f64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_double
    PP = ctypes.POINTER(ctypes.c_void_p)
    sigs = {
        "kde_abi_version": (i32, []),
        "kde_last_error": (ctypes.c_char_p, []),
        "kde_status_string": (ctypes.c_char_p, [ctypes.c_int]),
        "kde_create": (ctypes.c_int, [P, i64, i32, P, PP]),
        "kde_create_sharded": (ctypes.c_int, [P, i64, i64, i64, i32, P, P, i32, i32, PP]),
        "kde_get_unique_id": (ctypes.c_int, [P]),
        "kde_create_sharded_peer": (ctypes.c_int, [P, i64, i64, i64, i32, P, i32, i32, PP]),
        "kde_peer_handle": (ctypes.c_int, [P, P]),
        "kde_peer_attach": (ctypes.c_int, [P, P]),
        "kde_destroy": (None, [P]),
        "kde_get_info": (ctypes.c_int, [P, P, P, P, P, P]),
        "kde_get_bandwidth": (ctypes.c_int, [P, P]),
        "kde_set_bandwidth": (ctypes.c_int, [P, P]),
        "kde_set_retain": (ctypes.c_int, [P, i32]),
        "kde_set_kernel": (ctypes.c_int, [P, i32]),
        "kde_get_kernel": (ctypes.c_int, [P, P]),
        "kde_set_cull": (ctypes.c_int, [P, i32]),
        "kde_get_cull": (ctypes.c_int, [P, P]),
        "kde_set_cells": (ctypes.c_int, [P, i32]),
        "kde_get_cells": (ctypes.c_int, [P, P, P, P]),
        "kde_estimate_batch": (ctypes.c_int, [P, P, P, i64, P, P]),
        "kde_estimate_batch_dev": (ctypes.c_int, [P, P, P, i64, P, P, P]),
        "kde_loss_and_grad": (ctypes.c_int, [P, P, P, P, i64, i32, f64, i32, P, P, P]),
        "kde_loss_and_grad_dev": (ctypes.c_int, [P, P, P, P, i64, i32, f64, i32, P, P, P, P]),
        "kde_karma_update": (ctypes.c_int, [P, P, P, f64, ctypes.POINTER(KarmaParams), P, i64, P]),
        "kde_online_update": (ctypes.c_int, [P, P, P, f64, ctypes.POINTER(OnlineParams), P]),
        "kde_replace_points": (ctypes.c_int, [P, P, P, i64, f64]),
        "kde_reservoir_select": (ctypes.c_int, [ctypes.c_uint64, i64, i64, i64, P]),
        "kde_insert_rows": (ctypes.c_int, [P, P, i64, ctypes.c_uint64, P, f64, P]),
        "kde_insert_rows_async": (ctypes.c_int, [P, P, i64, ctypes.c_uint64, P, f64, P, P]),
        "kde_get_karma": (ctypes.c_int, [P, P]),
        "kde_set_karma": (ctypes.c_int, [P, P]),
        "kde_get_sample": (ctypes.c_int, [P, P]),
        "kde_get_contributions": (ctypes.c_int, [P, P]),
        "kde_get_online_state": (ctypes.c_int, [P, P, P, P, P, P]),
        "kde_set_online_state": (ctypes.c_int, [P, P, P, P, P, i32]),
        "kde_synchronize": (ctypes.c_int, [P]),
        "kde_count_in_box_dev": (ctypes.c_int, [P, i64, i32, P, P, i64, P, P]),
        "kde_set_profiling": (ctypes.c_int, [P, i32]),
        "kde_get_profile": (ctypes.c_int, [P, P, P, P]),
        "kde_karma_update_dev": (ctypes.c_int, [P, P, P, P, ctypes.POINTER(KarmaParams), P, i64, P, P]),
        "kde_online_update_dev": (ctypes.c_int, [P, P, ctypes.POINTER(OnlineParams), P]),
        "kde_replace_points_dev": (ctypes.c_int, [P, P, P, P, i64, f64, P]),
        "kde_stream_step_dev": (ctypes.c_int, [P, P, P, P, ctypes.POINTER(KarmaParams), ctypes.POINTER(OnlineParams),
                                               P, i64, P, P, f64, P, P, P]),
    }
    for name, (res, args) in sigs.items():
        fn = getattr(L, name)
        fn.restype = res
        fn.argtypes = args
    _lib = L
    return L


def _check(st: int, allow=()):
    if st != KDE_OK and st not in allow:
        raise KDEError(st, lib().kde_last_error().decode(errors="replace"))
    return st


def _f32(a, shape=None):
    a = np.ascontiguousarray(a, dtype=np.float32)
    if shape is not None:
        a = a.reshape(shape)
    return a


def _f64(a):
    return np.ascontiguousarray(a, dtype=np.float64)


def _p(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _tp(t, dtype=None, numel=None, name="tensor"):
    """Device pointer of a torch tensor (plumbing only).  The C side cannot see
    dtype, layout or extent, so they are checked here: a CUDA tensor, contiguous,
    of the expected dtype ("f32" / "f64" / "i64") and with at least `numel` elements."""
    if t is None:
        return None
    if not getattr(t, "is_cuda", False):
        raise KDEError(KDE_EINVAL, f"{name} must be a CUDA tensor")
    if not t.is_contiguous():
        raise KDEError(KDE_EINVAL, f"{name} must be contiguous")
    if dtype is not None:
        want = {"f32": "torch.float32", "f64": "torch.float64", "i64": "torch.int64"}[dtype]
        if str(t.dtype) != want:
            raise KDEError(KDE_EINVAL, f"{name} must be {want}, got {t.dtype}")
    if numel is not None and t.numel() < numel:
        raise KDEError(KDE_EINVAL, f"{name} has {t.numel()} elements, needs >= {numel}")
    return ctypes.c_void_p(t.data_ptr())


def _dim(m) -> int:
    return kde_get_info(m)["d"]


def _bounds(d_lo, d_hi, d, q=None):
    """(q, d) fp32 device bounds of identical shape; returns q."""
    if d_lo.shape != d_hi.shape:
        raise KDEError(KDE_EINVAL, "lo and hi must have the same shape")
    if d_lo.numel() % d != 0 or (q is not None and d_lo.numel() != q * d):
        raise KDEError(KDE_EINVAL, f"bounds must hold q x {d} values, got shape {tuple(d_lo.shape)}")
    return d_lo.numel() // d


_CUDA_STREAM_LEGACY = 1  # cudaStreamLegacy: the C ABI reads a NULL stream as "the model's own stream"


def _stream_ptr(stream):
    """None -> NULL (the model's stream); a torch stream -> its handle, the default (legacy) stream,
    whose handle is 0, as cudaStreamLegacy so that the work is ordered with torch's default stream."""
    if stream is None:
        return None
    h = stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)
    return ctypes.c_void_p(h if h else _CUDA_STREAM_LEGACY)


# ---------------------------------------------------------------- C-ABI mirrors
def kde_create(sample, h=None):
    """kde_create: sample [n, d] (row-major fp32); h [d] or None (Scott, eq. 3)."""
    sample = _f32(sample)
    n, d = sample.shape
    hh = None if h is None else _f64(h)
    out = ctypes.c_void_p()
    _check(lib().kde_create(_p(sample), n, d, _p(hh), ctypes.byref(out)))
    return out


def kde_get_unique_id() -> bytes:
    buf = (ctypes.c_char * KDE_NCCL_ID_BYTES)()
    _check(lib().kde_get_unique_id(buf))
    return bytes(buf)


def kde_create_sharded(local_rows, row_offset: int, n_global: int, h, nccl_id: bytes, rank: int, world: int):
    local_rows = _f32(local_rows)
    n, d = local_rows.shape
    hh = None if h is None else _f64(h)
    idb = ctypes.create_string_buffer(nccl_id, KDE_NCCL_ID_BYTES) if nccl_id is not None else None
    out = ctypes.c_void_p()
    _check(lib().kde_create_sharded(_p(local_rows), n, row_offset, n_global, d, _p(hh), idb, rank, world,
                                    ctypes.byref(out)))
    return out


def kde_create_sharded_peer(local_rows, row_offset: int, n_global: int, h, rank: int, world: int):
    """Phase 1 of a peer-transport sharded model (kde_peer_handle / kde_peer_attach follow)."""
    local_rows = _f32(local_rows)
    n, d = local_rows.shape
    hh = None if h is None else _f64(h)
    out = ctypes.c_void_p()
    _check(lib().kde_create_sharded_peer(_p(local_rows), n, row_offset, n_global, d, _p(hh), rank, world,
                                         ctypes.byref(out)))
    return out


def kde_peer_handle(m) -> bytes:
    buf = (ctypes.c_char * KDE_PEER_HANDLE_BYTES)()
    _check(lib().kde_peer_handle(m, buf))
    return bytes(buf)


def kde_peer_attach(m, handles: bytes):
    buf = ctypes.create_string_buffer(handles, len(handles))
    _check(lib().kde_peer_attach(m, buf))


def kde_destroy(m):
    lib().kde_destroy(m)


def kde_get_info(m):
    nl, ng, d, r, w = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
    _check(lib().kde_get_info(m, ctypes.byref(nl), ctypes.byref(ng), ctypes.byref(d), ctypes.byref(r),
                              ctypes.byref(w)))
    return dict(n_local=nl.value, n_global=ng.value, d=d.value, rank=r.value, world=w.value)


def kde_get_bandwidth(m, d):
    h = np.empty(d, dtype=np.float64)
    _check(lib().kde_get_bandwidth(m, _p(h)))
    return h


def kde_set_bandwidth(m, h):
    h = _f64(h)
    _check(lib().kde_set_bandwidth(m, _p(h)))


def kde_set_kernel(m, kernel: int):
    _check(lib().kde_set_kernel(m, int(kernel)))


def kde_get_kernel(m) -> int:
    k = ctypes.c_int32()
    _check(lib().kde_get_kernel(m, ctypes.byref(k)))
    return k.value


def kde_set_cull(m, on: bool):
    _check(lib().kde_set_cull(m, int(bool(on))))


def kde_get_cull(m) -> bool:
    k = ctypes.c_int32()
    _check(lib().kde_get_cull(m, ctypes.byref(k)))
    return bool(k.value)


def kde_set_cells(m, on: bool):
    _check(lib().kde_set_cells(m, int(bool(on))))


def kde_get_cells(m, stats=False):
    """(on, index builds so far[, profiling counters: items, full items, points evaluated,
    points classified -- read and reset])"""
    k = ctypes.c_int32()
    b = ctypes.c_int64()
    st = (ctypes.c_int64 * 4)()
    _check(lib().kde_get_cells(m, ctypes.byref(k), ctypes.byref(b), st if stats else None))
    return (bool(k.value), b.value, list(st)) if stats else (bool(k.value), b.value)


def kde_set_retain(m, on: bool):
    _check(lib().kde_set_retain(m, int(bool(on))))


def kde_estimate_batch(m, lo, hi, d, grad=False):
    """est[q] (eq. 2+13) and, with grad, dp_hat/dh [q, d] (eq. 17)."""
    lo = _f32(lo).reshape(-1, d)
    hi = _f32(hi).reshape(-1, d)
    q = lo.shape[0]
    est = np.empty(q, dtype=np.float64)
    g = np.empty((q, d), dtype=np.float64) if grad else None
    _check(lib().kde_estimate_batch(m, _p(lo), _p(hi), q, _p(est), _p(g)))
    return (est, g) if grad else est


def kde_estimate_batch_dev(m, d_lo, d_hi, d_est, d_dpdh=None, stream=None):
    """Device-pointer variant (torch CUDA tensors; plumbing only): enqueue only."""
    d = _dim(m)
    q = _bounds(d_lo, d_hi, d)
    _check(lib().kde_estimate_batch_dev(m, _tp(d_lo, "f32", name="d_lo"), _tp(d_hi, "f32", name="d_hi"), q,
                                        _tp(d_est, "f64", q, "d_est"), _tp(d_dpdh, "f64", q * d, "d_dpdh"),
                                        _stream_ptr(stream)))


def kde_loss_and_grad(m, lo, hi, true_sel, d, loss=LOSS_SQUARED, lam=0.0, log_bandwidth=False, return_est=False):
    """(loss, grad[d]) of eq. (5)/(14)/(18) over the q boxes."""
    lo = _f32(lo).reshape(-1, d)
    hi = _f32(hi).reshape(-1, d)
    q = lo.shape[0]
    ts = _f64(true_sel)
    lo_ = ctypes.c_double()
    g = np.empty(d, dtype=np.float64)
    est = np.empty(q, dtype=np.float64) if return_est else None
    _check(lib().kde_loss_and_grad(m, _p(lo), _p(hi), _p(ts), q, loss, lam, int(bool(log_bandwidth)),
                                   ctypes.byref(lo_), _p(g), _p(est)))
    return (lo_.value, g, est) if return_est else (lo_.value, g)


def kde_loss_and_grad_dev(m, d_lo, d_hi, d_true, d_loss, d_grad, loss=LOSS_SQUARED, lam=0.0, log_bandwidth=False,
                          d_est=None, stream=None):
    d = _dim(m)
    q = _bounds(d_lo, d_hi, d)
    _check(lib().kde_loss_and_grad_dev(m, _tp(d_lo, "f32", name="d_lo"), _tp(d_hi, "f32", name="d_hi"),
                                       _tp(d_true, "f64", q, "d_true"), q, loss, lam,
                                       int(bool(log_bandwidth)), _tp(d_loss, "f64", 1, "d_loss"),
                                       _tp(d_grad, "f64", d, "d_grad"), _tp(d_est, "f64", q, "d_est"),
                                       _stream_ptr(stream)))


def kde_karma_update(m, lo, hi, true_sel: float, params: KarmaParams, cap: int):
    """Returns (ascending global indices of flagged points, total flagged)."""
    lo = _f32(lo).ravel()
    hi = _f32(hi).ravel()
    idx = np.empty(max(cap, 1), dtype=np.int64)
    nf = ctypes.c_int64()
    st = _check(lib().kde_karma_update(m, _p(lo), _p(hi), float(true_sel), ctypes.byref(params), _p(idx), cap,
                                       ctypes.byref(nf)), allow=(KDE_ETRUNC,))
    return idx[:min(nf.value, cap)].copy(), nf.value, st == KDE_ETRUNC


def kde_online_update(m, lo, hi, true_sel: float, params: OnlineParams) -> bool:
    lo = _f32(lo).ravel()
    hi = _f32(hi).ravel()
    upd = ctypes.c_int32()
    _check(lib().kde_online_update(m, _p(lo), _p(hi), float(true_sel), ctypes.byref(params), ctypes.byref(upd)))
    return bool(upd.value)


def kde_karma_update_dev(m, d_lo, d_hi, d_true, params: KarmaParams, d_idx, d_count, stream=None):
    """Device-resident karma pass (single GPU): enqueue only."""
    _bounds(d_lo, d_hi, _dim(m), 1)
    _check(lib().kde_karma_update_dev(m, _tp(d_lo, "f32", name="d_lo"), _tp(d_hi, "f32", name="d_hi"),
                                      _tp(d_true, "f64", 1, "d_true"), ctypes.byref(params),
                                      _tp(d_idx, "i64", name="d_idx"), d_idx.numel(),
                                      _tp(d_count, "i64", 1, "d_count"), _stream_ptr(stream)))


def kde_online_update_dev(m, d_true, params: OnlineParams, stream=None):
    _check(lib().kde_online_update_dev(m, _tp(d_true, "f64", 1, "d_true"), ctypes.byref(params),
                                       _stream_ptr(stream)))


def kde_replace_points_dev(m, d_idx, d_rows, d_count, k_init=0.0, stream=None):
    """Rows d_rows[r] -> global index d_idx[r] for r < min(d_count, len(d_idx))."""
    d = _dim(m)
    if d_rows.dim() != 2 or d_rows.shape[1] != d:
        raise KDEError(KDE_EINVAL, f"d_rows must be (k, {d}), got {tuple(d_rows.shape)}")
    _check(lib().kde_replace_points_dev(m, _tp(d_idx, "i64", name="d_idx"),
                                        _tp(d_rows, "f32", d_idx.numel() * d, "d_rows"),
                                        _tp(d_count, "i64", 1, "d_count"), d_idx.numel(), float(k_init),
                                        _stream_ptr(stream)))


def kde_stream_step_dev(m, d_lo, d_hi, d_true, kparams: KarmaParams, oparams, d_idx, d_count, d_rows, d_est,
                        d_dpdh, k_init=0.0, stream=None):
    """One device-resident streaming step (estimate + gradient + karma +
    Listing 1 + replacement) in three kernels; enqueue only."""
    d = _dim(m)
    _bounds(d_lo, d_hi, d, 1)
    if d_rows is not None and (d_rows.dim() != 2 or d_rows.shape[1] != d):
        raise KDEError(KDE_EINVAL, f"d_rows must be (k, {d}), got {tuple(d_rows.shape)}")
    _check(lib().kde_stream_step_dev(m, _tp(d_lo, "f32", name="d_lo"), _tp(d_hi, "f32", name="d_hi"),
                                     _tp(d_true, "f64", 1, "d_true"), ctypes.byref(kparams),
                                     None if oparams is None else ctypes.byref(oparams),
                                     _tp(d_idx, "i64", name="d_idx"), d_idx.numel(),
                                     _tp(d_count, "i64", 1, "d_count"),
                                     _tp(d_rows, "f32", d_idx.numel() * d, "d_rows"), float(k_init),
                                     _tp(d_est, "f64", 1, "d_est"),
                                     _tp(d_dpdh, "f64", d if oparams is not None else None, "d_dpdh"),
                                     _stream_ptr(stream)))


def kde_replace_points(m, idx, rows, k_init=0.0):
    idx = np.ascontiguousarray(idx, dtype=np.int64)
    rows = _f32(rows)
    _check(lib().kde_replace_points(m, _p(idx), _p(rows), len(idx), float(k_init)))


def kde_reservoir_select(seed: int, n_sample: int, n_seen: int, k: int) -> np.ndarray:
    """Algorithm R decisions of the host: slot per arrival n_seen+1 .. n_seen+k, or -1."""
    out = np.empty(max(k, 1), dtype=np.int64)
    _check(lib().kde_reservoir_select(seed, n_sample, n_seen, k, _p(out)))
    return out[:k]


def kde_insert_rows(m, rows, seed: int, n_seen: int, k_init=0.0):
    """Insert k rows through the reservoir; returns (new n_seen, slots written)."""
    rows = _f32(rows)
    ns = ctypes.c_int64(n_seen)
    nw = ctypes.c_int64()
    _check(lib().kde_insert_rows(m, _p(rows), rows.shape[0], seed, ctypes.byref(ns), float(k_init),
                                 ctypes.byref(nw)))
    return ns.value, nw.value


def kde_insert_rows_async(m, rows, seed: int, n_seen: int, k_init=0.0, stream=None):
    """kde_insert_rows with the device work enqueued on `stream` (no wait); returns (new n_seen, slots written)."""
    rows = _f32(rows)
    ns = ctypes.c_int64(n_seen)
    nw = ctypes.c_int64()
    _check(lib().kde_insert_rows_async(m, _p(rows), rows.shape[0], seed, ctypes.byref(ns), float(k_init),
                                       ctypes.byref(nw), _stream_ptr(stream)))
    return ns.value, nw.value


def kde_get_karma(m, n):
    k = np.empty(n, dtype=np.float64)
    _check(lib().kde_get_karma(m, _p(k)))
    return k


def kde_set_karma(m, karma):
    k = _f64(karma)
    _check(lib().kde_set_karma(m, _p(k)))


def kde_get_sample(m, n, d):
    r = np.empty((n, d), dtype=np.float32)
    _check(lib().kde_get_sample(m, _p(r)))
    return r


def kde_get_contributions(m, n):
    c = np.empty(n, dtype=np.float32)
    _check(lib().kde_get_contributions(m, _p(c)))
    return c


def kde_get_online_state(m, d):
    a, s, l_, g = (np.empty(d) for _ in range(4))
    cnt = ctypes.c_int32()
    _check(lib().kde_get_online_state(m, _p(a), _p(s), _p(l_), _p(g), ctypes.byref(cnt)))
    return dict(acc=a, ms=s, lr=l_, gprev=g, count=cnt.value)


def kde_set_online_state(m, acc, ms, lr, gprev, count):
    a, s, l_, g = _f64(acc), _f64(ms), _f64(lr), _f64(gprev)
    _check(lib().kde_set_online_state(m, _p(a), _p(s), _p(l_), _p(g), int(count)))


def kde_synchronize(m):
    _check(lib().kde_synchronize(m))


def kde_set_profiling(m, on: bool):
    _check(lib().kde_set_profiling(m, int(bool(on))))


def kde_get_profile(m):
    """(summed scan-kernel ms, scan launches, all kernel launches) since the last reset."""
    ms, sl, al = ctypes.c_double(), ctypes.c_int64(), ctypes.c_int64()
    _check(lib().kde_get_profile(m, ctypes.byref(ms), ctypes.byref(sl), ctypes.byref(al)))
    return ms.value, sl.value, al.value


def kde_count_in_box_dev(d_rows, d_lo, d_hi, d_counts, stream=None):
    """Harness only: exact counts of rows of R in each open box (the DBMS feedback)."""
    n, d = d_rows.shape
    q = _bounds(d_lo, d_hi, d)
    _check(lib().kde_count_in_box_dev(_tp(d_rows, "f32", name="d_rows"), n, d, _tp(d_lo, "f32", name="d_lo"),
                                      _tp(d_hi, "f32", name="d_hi"), q, _tp(d_counts, "i64", q, "d_counts"),
                                      _stream_ptr(stream)))


# ---------------------------------------------------------------- convenience wrapper
@dataclass
class KDEModel:
    """Owns a kde_model handle.  Methods map 1:1 to the C ABI."""
    handle: ctypes.c_void_p
    n: int
    n_global: int
    d: int
    rank: int = 0
    world: int = 1

    @classmethod
    def create(cls, sample, h=None):
        sample = _f32(sample)
        hd = kde_create(sample, h)
        n, d = sample.shape
        return cls(hd, n, n, d)

    @classmethod
    def create_sharded(cls, local_rows, row_offset, n_global, h, nccl_id, rank, world):
        hd = kde_create_sharded(local_rows, row_offset, n_global, h, nccl_id, rank, world)
        info = kde_get_info(hd)
        return cls(hd, info["n_local"], info["n_global"], info["d"], rank, world)

    @classmethod
    def create_sharded_peer(cls, local_rows, row_offset, n_global, h, rank, world, all_gather_bytes):
        """Peer-transport sharded model; all_gather_bytes(b: bytes) -> list of every rank's bytes
        (host bootstrap, e.g. torch.distributed.all_gather_object)."""
        hd = kde_create_sharded_peer(local_rows, row_offset, n_global, h, rank, world)
        try:
            if world > 1:
                kde_peer_attach(hd, b"".join(all_gather_bytes(kde_peer_handle(hd))))
        except Exception:
            kde_destroy(hd)
            raise
        info = kde_get_info(hd)
        return cls(hd, info["n_local"], info["n_global"], info["d"], rank, world)

    def close(self):
        if self.handle:
            kde_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    @property
    def bandwidth(self):
        return kde_get_bandwidth(self.handle, self.d)

    @bandwidth.setter
    def bandwidth(self, h):
        kde_set_bandwidth(self.handle, h)

    def set_kernel(self, kernel):
        """KERNEL_GAUSSIAN (paper, default) or KERNEL_EPANECHNIKOV (or 'gauss' / 'epan')."""
        if isinstance(kernel, str):
            kernel = {"gauss": KERNEL_GAUSSIAN, "epan": KERNEL_EPANECHNIKOV}[kernel]
        kde_set_kernel(self.handle, kernel)

    @property
    def kernel(self):
        return kde_get_kernel(self.handle)

    def set_retain(self, on=True):
        kde_set_retain(self.handle, on)

    @property
    def cull(self):
        """single-box scan skips points whose contribution is provably < 2^-64 (default on)"""
        return kde_get_cull(self.handle)

    @cull.setter
    def cull(self, on):
        kde_set_cull(self.handle, on)

    @property
    def cells(self):
        """culled batched scan over the spatially ordered copy of the sample (default on, DESIGN R17)"""
        return kde_get_cells(self.handle)[0]

    @cells.setter
    def cells(self, on):
        kde_set_cells(self.handle, on)

    def estimate(self, lo, hi, grad=False):
        return kde_estimate_batch(self.handle, lo, hi, self.d, grad)

    def loss_and_grad(self, lo, hi, true_sel, loss=LOSS_SQUARED, lam=0.0, log_bandwidth=False, return_est=False):
        return kde_loss_and_grad(self.handle, lo, hi, true_sel, self.d, loss, lam, log_bandwidth, return_est)

    def karma_update(self, lo, hi, true_sel, params=None, cap=None):
        params = params or karma_params()
        return kde_karma_update(self.handle, lo, hi, true_sel, params, self.n_global if cap is None else cap)

    def online_update(self, lo, hi, true_sel, params=None):
        return kde_online_update(self.handle, lo, hi, true_sel, params or online_params())

    def replace_points(self, idx, rows, k_init=0.0):
        kde_replace_points(self.handle, idx, rows, k_init)

    def insert_rows(self, rows, seed, n_seen, k_init=0.0):
        """Reservoir inserts: returns (new n_seen, slots written)."""
        return kde_insert_rows(self.handle, rows, seed, n_seen, k_init)

    @property
    def karma(self):
        return kde_get_karma(self.handle, self.n)

    @karma.setter
    def karma(self, k):
        kde_set_karma(self.handle, k)

    @property
    def sample(self):
        return kde_get_sample(self.handle, self.n, self.d)

    def contributions(self):
        return kde_get_contributions(self.handle, self.n)

    def online_state(self):
        return kde_get_online_state(self.handle, self.d)

    def synchronize(self):
        kde_synchronize(self.handle)

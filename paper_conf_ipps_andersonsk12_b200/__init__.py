"""paper_conf_ipps_andersonsk12_b200 -- B200-native batched Householder QR.

Thin Python binding (argument marshalling only) over the C ABI of
``libbqr.so`` (declared in ``include/bqr.h``); every step of the
factorisation runs in the library's hand-written sm_100a kernels.  There is
no CPU or PyTorch fallback: if the shared library is missing or cannot be
loaded, every call raises.

Operation: LAPACK xGEQRF / xORGQR / xORMQR('L','C') semantics for batches of
small matrices, fp32 and complex64.

Tensor convention: a batch of m x n matrices is a CUDA tensor of shape
(batch, m, n) stored column-major per matrix, i.e. strides
(lda*n, 1, lda) with lda >= m -- the layout ``torch.geqrf`` uses.  Use
:func:`colmajor` to obtain one from any tensor.  Calls are asynchronous on
``torch.cuda.current_stream()`` (or the given stream).
"""
from __future__ import annotations

import ctypes
import os

__all__ = [
    "load", "colmajor", "geqrf_batched", "orgqr_batched", "apply_qh_batched",
    "geqrf_batched_host", "host_workspace_bytes", "kernel_name", "geqrf_launches",
    "BQRError", "R32", "C64", "lib_path", "geqrf_batched_ptr", "geqrf_qhb_batched", "gels_batched",
    "getrf_np_batched", "gauss_jordan_batched",
]

R32, C64 = 0, 1
_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libbqr.so")
_lib = None


class BQRError(RuntimeError):
    pass


def lib_path() -> str:
    return _LIB_PATH


def load():
    """Load libbqr.so (built by build.py / __graft_entry__.build()).  Raises
    if it is absent: there is no fallback path."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIB_PATH):
        raise BQRError(f"{_LIB_PATH} not found: run `python -m paper_conf_ipps_andersonsk12_b200.build` "
                       "(the CUDA library is required; there is no CPU fallback)")
    lib = ctypes.CDLL(_LIB_PATH)
    i, p, sz = ctypes.c_int, ctypes.c_void_p, ctypes.c_size_t
    lib.bqr_geqrf_batched.argtypes = [i, i, i, i, p, i, p, p]
    lib.bqr_orgqr_batched.argtypes = [i, i, i, i, i, p, i, p, p]
    lib.bqr_apply_qh_batched.argtypes = [i, i, i, i, i, i, p, i, p, p, i, p]
    if hasattr(lib, "bqr_geqrf_qhb_batched"):  # absent in pre-fusion builds (A/B timing)
        lib.bqr_geqrf_qhb_batched.argtypes = [i, i, i, i, i, p, i, p, p, i, p]
        lib.bqr_geqrf_qhb_batched.restype = i
        lib.bqr_qhb_kernel_name.argtypes = [i, i, i, i]
        lib.bqr_qhb_kernel_name.restype = ctypes.c_char_p
    if hasattr(lib, "bqr_gels_batched"):  # absent in older builds (A/B timing)
        lib.bqr_gels_batched.argtypes = [i, i, i, i, i, p, i, p, p, i, p, p]
        lib.bqr_gels_batched.restype = i
    if hasattr(lib, "bqr_getrf_np_batched"):  # NEXT-3 (absent in older builds)
        lib.bqr_getrf_np_batched.argtypes = [i, i, i, i, p, i, p, p]
        lib.bqr_getrf_np_batched.restype = i
        lib.bqr_gauss_jordan_batched.argtypes = [i, i, i, i, p, i, p, i, p, p]
        lib.bqr_gauss_jordan_batched.restype = i
    if hasattr(lib, "bqr_lu_kernel_name"):
        lib.bqr_lu_kernel_name.argtypes = [i, i, i, i, i]
        lib.bqr_lu_kernel_name.restype = ctypes.c_char_p
    lib.bqr_geqrf_batched_host.argtypes = [i, i, i, i, p, i, p, p, sz, p]
    lib.bqr_host_workspace_bytes.argtypes = [i, i, i, i, i]
    lib.bqr_host_workspace_bytes.restype = sz
    for f in ("bqr_geqrf_batched", "bqr_orgqr_batched", "bqr_apply_qh_batched", "bqr_geqrf_batched_host"):
        getattr(lib, f).restype = i
    lib.bqr_status_string.argtypes = [i]
    lib.bqr_status_string.restype = ctypes.c_char_p
    lib.bqr_kernel_name.argtypes = [i, i, i]
    lib.bqr_kernel_name.restype = ctypes.c_char_p
    if hasattr(lib, "bqr_geqrf_wy_batched"):  # compact-WY blocked variant (absent in older builds)
        lib.bqr_geqrf_wy_batched.argtypes = [i, i, i, i, p, i, p, p, sz, p]
        lib.bqr_geqrf_wy_batched.restype = i
        lib.bqr_geqrf_wy_workspace_bytes.argtypes = [i, i, i, i, i]
        lib.bqr_geqrf_wy_workspace_bytes.restype = sz
        lib.bqr_geqrf_wy_kernel_name.argtypes = [i, i, i, i]
        lib.bqr_geqrf_wy_kernel_name.restype = ctypes.c_char_p
    if hasattr(lib, "bqr_resident_matrices"):  # (older builds, e.g. A/B libraries, lack the diagnostics)
        lib.bqr_resident_matrices.argtypes = [i, i, i]
        lib.bqr_resident_matrices.restype = ctypes.c_longlong
        lib.bqr_class_count.argtypes = []
        lib.bqr_class_count.restype = i
        ip = ctypes.POINTER(ctypes.c_int)
        lib.bqr_class_info.argtypes = [i, ip, ip, ip, ip, ip, ip]
        lib.bqr_class_info.restype = ctypes.c_char_p
    lib.bqr_geqrf_launches.argtypes = [i, i, i, i]
    lib.bqr_geqrf_launches.restype = i
    lib.bqr_version.restype = ctypes.c_char_p
    _lib = lib
    return lib


def _check(status: int, what: str):
    if status != 0:
        msg = load().bqr_status_string(status).decode()
        raise BQRError(f"{what} failed: status {status} ({msg})")


def _dtype_code(t) -> int:
    import torch
    if t.dtype == torch.float32:
        return R32
    if t.dtype == torch.complex64:
        return C64
    raise TypeError(f"unsupported dtype {t.dtype}: float32 or complex64")


def _stream_ptr(stream):
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def colmajor(A, lda: int | None = None):
    """Copy A (batch, m, n) into column-major-per-matrix storage with leading
    dimension lda (>= m); returns the (batch, m, n) view."""
    import torch
    batch, m, n = A.shape
    lda = m if lda is None else lda
    buf = torch.empty((batch, n, lda), dtype=A.dtype, device=A.device)
    view = buf.transpose(1, 2)[:, :m, :]
    view.copy_(A)
    return view


def _layout(A):
    """(m, n, lda) of a column-major (batch, m, n) tensor, validating strides."""
    if A.dim() != 3:
        raise ValueError("expected a (batch, m, n) tensor")
    batch, m, n = A.shape
    s0, s1, s2 = A.stride()
    lda = s2 if n > 1 else max(m, 1)
    if (m > 1 and s1 != 1) or (batch > 1 and s0 != lda * n) or lda < max(1, m):
        raise ValueError(f"A must be column-major per matrix with strides (lda*n, 1, lda); got {A.stride()}")
    return m, n, lda


def geqrf_batched(A, tau=None, stream=None):
    """In-place batched QR: A <- [R; V], returns (A, tau).  LAPACK xGEQRF."""
    import torch
    if not A.is_cuda:
        raise ValueError("A must be a CUDA tensor (use geqrf_batched_host for host buffers)")
    batch, m, n = A.shape
    m, n, lda = _layout(A)
    k = min(m, n)
    if tau is None:
        tau = torch.empty((batch, k), dtype=A.dtype, device=A.device)
    st = load().bqr_geqrf_batched(_dtype_code(A), m, n, batch, ctypes.c_void_p(A.data_ptr()), lda,
                                  ctypes.c_void_p(tau.data_ptr()), _stream_ptr(stream))
    _check(st, "bqr_geqrf_batched")
    return A, tau


def geqrf_batched_ptr(dtype: int, m: int, n: int, batch: int, A_ptr: int, lda: int, tau_ptr: int,
                      stream_ptr: int = 0) -> int:
    """Raw C-ABI call (device pointers as ints); returns the status code."""
    return load().bqr_geqrf_batched(dtype, m, n, batch, ctypes.c_void_p(A_ptr), lda,
                                    ctypes.c_void_p(tau_ptr), ctypes.c_void_p(stream_ptr))


def orgqr_batched(A, tau, n: int | None = None, stream=None):
    """In-place: A (batch, m, n) <- first n columns of Q from reflectors + tau."""
    batch, m, ncols = A.shape
    m, ncols, lda = _layout(A)
    k = tau.shape[-1]
    st = load().bqr_orgqr_batched(_dtype_code(A), m, ncols, k, batch, ctypes.c_void_p(A.data_ptr()), lda,
                                  ctypes.c_void_p(tau.data_ptr()), _stream_ptr(stream))
    _check(st, "bqr_orgqr_batched")
    return A


def apply_qh_batched(A, tau, B, stream=None):
    """In-place: B (batch, m, nrhs) <- Q^H B with Q from (A, tau)."""
    batch, m, n = A.shape
    m, n, lda = _layout(A)
    _, mb, nrhs = B.shape
    _, _, ldb = _layout(B)
    k = tau.shape[-1]
    st = load().bqr_apply_qh_batched(_dtype_code(A), m, n, k, nrhs, batch, ctypes.c_void_p(A.data_ptr()), lda,
                                     ctypes.c_void_p(tau.data_ptr()), ctypes.c_void_p(B.data_ptr()), ldb,
                                     _stream_ptr(stream))
    _check(st, "bqr_apply_qh_batched")
    return B


def geqrf_qhb_batched(A, B, tau=None, stream=None):
    """Fused: A <- [R; V] and B <- Q^H B in one kernel (the augmented [A | b]
    of P:L313).  Returns (A, tau, B)."""
    import torch
    batch, m, n = A.shape
    m, n, lda = _layout(A)
    _, mb, nrhs = B.shape
    _, _, ldb = _layout(B)
    k = min(m, n)
    if tau is None:
        tau = torch.empty((batch, k), dtype=A.dtype, device=A.device)
    st = load().bqr_geqrf_qhb_batched(_dtype_code(A), m, n, nrhs, batch, ctypes.c_void_p(A.data_ptr()), lda,
                                      ctypes.c_void_p(tau.data_ptr()), ctypes.c_void_p(B.data_ptr()), ldb,
                                      _stream_ptr(stream))
    _check(st, "bqr_geqrf_qhb_batched")
    return A, tau, B


def gels_batched(A, B, tau=None, info=None, stream=None):
    """Least squares by QR: A (batch, m, n) <- [R; V],
    B (batch, m, nrhs) <- [X; residual components].  Returns (A, tau, B, info)
    with info (batch,) int32 on the device (0, or j+1 for a zero R_jj)."""
    import torch
    batch, m, n = A.shape
    m, n, lda = _layout(A)
    _, mb, nrhs = B.shape
    _, _, ldb = _layout(B)
    if tau is None:
        tau = torch.empty((batch, n), dtype=A.dtype, device=A.device)
    if info is None:
        info = torch.empty((batch,), dtype=torch.int32, device=A.device)
    st = load().bqr_gels_batched(_dtype_code(A), m, n, nrhs, batch, ctypes.c_void_p(A.data_ptr()), lda,
                                 ctypes.c_void_p(tau.data_ptr()), ctypes.c_void_p(B.data_ptr()), ldb,
                                 ctypes.c_void_p(info.data_ptr()), _stream_ptr(stream))
    _check(st, "bqr_gels_batched")
    return A, tau, B, info


def getrf_np_batched(A, info=None, stream=None):
    """LU without pivoting: A (batch, m, n) column-major per
    matrix <- L (strict lower) + U.  Returns (A, info) with info (batch,)
    int32 on the device (0, or k+1 for the first zero pivot)."""
    import torch
    batch = A.shape[0]
    m, n, lda = _layout(A)
    if info is None:
        info = torch.empty((batch,), dtype=torch.int32, device=A.device)
    st = load().bqr_getrf_np_batched(_dtype_code(A), m, n, batch, ctypes.c_void_p(A.data_ptr()), lda,
                                     ctypes.c_void_p(info.data_ptr()), _stream_ptr(stream))
    _check(st, "bqr_getrf_np_batched")
    return A, info


def gauss_jordan_batched(A, B, info=None, stream=None):
    """Gauss-Jordan without pivoting on [A | B]: A (batch, n, n)
    is destroyed, B (batch, n, nrhs) <- X.  Returns (A, B, info)."""
    import torch
    batch = A.shape[0]
    m, n, lda = _layout(A)
    _, nrhs, ldb = _layout(B)
    if info is None:
        info = torch.empty((batch,), dtype=torch.int32, device=A.device)
    st = load().bqr_gauss_jordan_batched(_dtype_code(A), n, nrhs, batch, ctypes.c_void_p(A.data_ptr()), lda,
                                         ctypes.c_void_p(B.data_ptr()), ldb, ctypes.c_void_p(info.data_ptr()),
                                         _stream_ptr(stream))
    _check(st, "bqr_gauss_jordan_batched")
    return A, B, info


def host_workspace_bytes(dtype: int, m: int, n: int, lda: int, chunk: int) -> int:
    return int(load().bqr_host_workspace_bytes(dtype, m, n, lda, chunk))


def geqrf_batched_host(dtype: int, m: int, n: int, batch: int, A_host_ptr: int, lda: int, tau_host_ptr: int,
                       workspace_ptr: int, workspace_bytes: int, stream=None) -> None:
    """Synchronous QR of a HOST batch streamed through a device workspace."""
    st = load().bqr_geqrf_batched_host(dtype, m, n, batch, ctypes.c_void_p(A_host_ptr), lda,
                                       ctypes.c_void_p(tau_host_ptr), ctypes.c_void_p(workspace_ptr),
                                       workspace_bytes, _stream_ptr(stream))
    _check(st, "bqr_geqrf_batched_host")


def geqrf_wy_workspace_bytes(dtype: int, m: int, n: int, lda: int, chunk: int) -> int:
    return int(load().bqr_geqrf_wy_workspace_bytes(dtype, m, n, lda, chunk))


def geqrf_wy_batched_ptr(dtype: int, m: int, n: int, batch: int, A_ptr: int, lda: int, tau_ptr: int,
                         work_ptr: int, work_bytes: int, stream=None) -> int:
    """Compact-WY blocked QR (tensor-core trailing updates) through the C ABI;
    returns the status code."""
    return load().bqr_geqrf_wy_batched(dtype, m, n, batch, ctypes.c_void_p(A_ptr), lda, ctypes.c_void_p(tau_ptr),
                                       ctypes.c_void_p(work_ptr), work_bytes, _stream_ptr(stream))


def size_classes() -> list:
    """The library's size-class table (bqr_class_info): one dict per entry
    with dtype, mmax, nmax, exact_m, exact_n, experiment, augmented,
    dispatched (picked by bqr_geqrf_batched) and name."""
    lib = load()
    out = []
    vals = [ctypes.c_int() for _ in range(6)]
    for idx in range(lib.bqr_class_count()):
        name = lib.bqr_class_info(idx, *[ctypes.byref(v) for v in vals])
        dt, mmax, nmax, em, en, fl = (v.value for v in vals)
        out.append({"name": name.decode(), "dtype": dt, "mmax": mmax, "nmax": nmax, "exact_m": em,
                    "exact_n": en, "experiment": bool(fl & 1), "augmented": bool(fl & 2),
                    "dispatched": not (fl & 4)})
    return out


def kernel_name(dtype: int, m: int, n: int) -> str:
    return load().bqr_kernel_name(dtype, m, n).decode()


def geqrf_launches(dtype: int, m: int, n: int, batch: int) -> int:
    return int(load().bqr_geqrf_launches(dtype, m, n, batch))

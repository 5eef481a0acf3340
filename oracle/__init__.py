"""oracle -- TEST INFRASTRUCTURE ONLY (parity oracle for the CUDA path).

Plain, slow, double-precision CPU Householder QR with LAPACK xGEQR2/xLARFG
semantics ("consistent with LAPACK", Sec. III-C; column steps
in the order of Table VI), plus xORG2R/xUNG2R (explicit Q) and
xORM2R/xUNM2R('L','C') (Q^H B, the least-squares step of Sec. III-D,
P:L309-313).  The arithmetic lives in ``bqr_ref.c``; this module only
compiles/loads it with ctypes and marshals numpy arrays.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  It
shares no code with ``paper_conf_ipps_andersonsk12_b200`` and never imports it.

Every public function here has pins in tests/test_oracle_*.py (closed forms,
LAPACK, invariants, brute force); nothing is "parity unpinned" except the
readings listed in DESIGN.md (sign-flip V/tau bits, Q6 scaling regimes).

Array convention (same as the product's Python binding): a batch of m x n
matrices is a numpy array ``A`` of shape (batch, m, n) holding the *logical*
matrices; ``*_cm`` functions take the raw column-major storage instead:
shape (batch, n, lda), element (b, row, col) at ``A_cm[b, col, row]``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "bqr_ref.c")
_SRCS = [_SRC, os.path.join(_HERE, "lu_ref.c")]  # lu_ref.c: NEXT-3 (LU / Gauss-Jordan)
_LIB = os.path.join(_HERE, "libbqr_ref.so")
_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile libbqr_ref.so with gcc -O2 -fopenmp (no -ffast-math: IEEE fp64)."""
    if force or not os.path.exists(_LIB) or any(os.path.getmtime(_LIB) < os.path.getmtime(s) for s in _SRCS):
        cmd = ["gcc", "-O2", "-std=c11", "-fopenmp", "-fPIC", "-shared",
               "-fno-fast-math", "-ffp-contract=off", "-o", _LIB, *_SRCS, "-lm"]
        subprocess.check_call(cmd)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_LIB)
            i, i64, p = ctypes.c_int, ctypes.c_int64, ctypes.c_void_p
            for name in ("bqr_ref_geqrf_d", "bqr_ref_geqrf_z"):
                getattr(lib, name).argtypes = [i, i, i64, p, i, p, p]
                getattr(lib, name).restype = None
            for name in ("bqr_ref_orgqr_d", "bqr_ref_orgqr_z"):
                getattr(lib, name).argtypes = [i, i, i, i64, p, i, p]
                getattr(lib, name).restype = None
            for name in ("bqr_ref_apply_qh_d", "bqr_ref_apply_qh_z"):
                getattr(lib, name).argtypes = [i, i, i, i, i64, p, i, p, p, i]
                getattr(lib, name).restype = None
            for name in ("bqr_ref_gels_d", "bqr_ref_gels_z"):
                getattr(lib, name).argtypes = [i, i, i, i64, p, i, p, p, i, p]
                getattr(lib, name).restype = None
            for name in ("bqr_ref_getrf_np_d", "bqr_ref_getrf_np_z"):
                getattr(lib, name).argtypes = [i, i, i64, p, i, p]
                getattr(lib, name).restype = None
            for name in ("bqr_ref_gauss_jordan_d", "bqr_ref_gauss_jordan_z"):
                getattr(lib, name).argtypes = [i, i, i64, p, i, p, i, p]
                getattr(lib, name).restype = None
            lib.bqr_ref_set_threads.argtypes = [i]
            lib.bqr_ref_max_threads.restype = i
            _lib = lib
    return _lib


def set_threads(n: int) -> None:
    """Number of OpenMP threads (0 = all cores available to the process)."""
    _load().bqr_ref_set_threads(int(n))


def max_threads() -> int:
    return int(_load().bqr_ref_max_threads())


def _is_complex(a: np.ndarray) -> bool:
    return np.iscomplexobj(a)


def _widen(a: np.ndarray) -> np.ndarray:
    """fp32 -> fp64 / c64 -> c128, exact."""
    return np.ascontiguousarray(a, dtype=np.complex128 if _is_complex(a) else np.float64)


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


# --------------------------------------------------------------------------
# raw column-major entry points
# --------------------------------------------------------------------------

def geqrf_cm(A_cm: np.ndarray, m: int, with_margin: bool = True):
    """In-place-style geqr2 on column-major storage (batch, n, lda).

    Returns (A_out_cm, tau (batch, k), margin (batch, k) or None)."""
    lib = _load()
    A = _widen(A_cm).copy()
    batch, n, lda = A.shape
    k = min(m, n)
    cplx = _is_complex(A)
    tau = np.zeros((batch, k), dtype=A.dtype)
    margin = np.ones((batch, k), dtype=np.float64) if with_margin else None
    if batch and m and n:
        fn = lib.bqr_ref_geqrf_z if cplx else lib.bqr_ref_geqrf_d
        fn(m, n, batch, _ptr(A), lda, _ptr(tau), _ptr(margin) if with_margin else None)
    return A, tau, margin


def orgqr_cm(A_cm: np.ndarray, m: int, k: int, tau: np.ndarray):
    lib = _load()
    A = _widen(A_cm).copy()
    batch, n, lda = A.shape
    t = np.ascontiguousarray(tau, dtype=A.dtype).reshape(batch, k)
    if batch and m and n:
        fn = lib.bqr_ref_orgqr_z if _is_complex(A) else lib.bqr_ref_orgqr_d
        fn(m, n, k, batch, _ptr(A), lda, _ptr(t))
    return A


def apply_qh_cm(A_cm: np.ndarray, m: int, k: int, tau: np.ndarray, B_cm: np.ndarray):
    """B (batch, nrhs, ldb) column-major <- Q^H B."""
    lib = _load()
    A = _widen(A_cm)
    batch, n, lda = A.shape
    B = np.ascontiguousarray(B_cm, dtype=A.dtype).copy()
    _, nrhs, ldb = B.shape
    t = np.ascontiguousarray(tau, dtype=A.dtype).reshape(batch, k)
    if batch and m and nrhs and k:
        fn = lib.bqr_ref_apply_qh_z if _is_complex(A) else lib.bqr_ref_apply_qh_d
        fn(m, n, k, nrhs, batch, _ptr(A), lda, _ptr(t), _ptr(B), ldb)
    return B


# --------------------------------------------------------------------------
# logical (batch, m, n) convenience API
# --------------------------------------------------------------------------

def to_cm(A: np.ndarray) -> np.ndarray:
    """(batch, m, n) logical -> (batch, n, m) column-major storage (lda = m)."""
    return np.ascontiguousarray(np.swapaxes(A, -1, -2))


def from_cm(A_cm: np.ndarray, m: int) -> np.ndarray:
    return np.ascontiguousarray(np.swapaxes(A_cm[..., :m], -1, -2))


def geqrf(A: np.ndarray, with_margin: bool = True):
    """A (batch, m, n) -> (RV (batch, m, n) fp64/c128, tau (batch, k), margin)."""
    A = np.asarray(A)
    if A.ndim == 2:
        A = A[None]
    m = A.shape[1]
    out, tau, margin = geqrf_cm(to_cm(A), m, with_margin)
    return from_cm(out, m), tau, margin


def orgqr(RV: np.ndarray, tau: np.ndarray, n: int | None = None):
    """First n columns of Q from the reflectors in RV (batch, m, >=k)."""
    RV = np.asarray(RV)
    batch, m, ncols = RV.shape
    k = tau.shape[-1]
    n = ncols if n is None else n
    W = np.zeros((batch, m, n), dtype=np.result_type(RV.dtype, np.float64))
    W[:, :, :min(n, ncols)] = RV[:, :, :min(n, ncols)]
    return from_cm(orgqr_cm(to_cm(W), m, k, tau), m)


def apply_qh(RV: np.ndarray, tau: np.ndarray, B: np.ndarray):
    """Q^H B with Q from (RV, tau); B (batch, m, nrhs)."""
    RV = np.asarray(RV)
    m = RV.shape[1]
    k = tau.shape[-1]
    return from_cm(apply_qh_cm(to_cm(RV), m, k, tau, to_cm(np.asarray(B))), m)


def triu_r(RV: np.ndarray) -> np.ndarray:
    """R = upper trapezoid of the geqrf output."""
    return np.triu(RV)


def gels_cm(A_cm: np.ndarray, m: int, B_cm: np.ndarray):
    """Least squares min ||A x - b|| by QR (paper Sec. III-D) on
    column-major storage: A (batch, n, lda), B (batch, nrhs, ldb), m >= n.
    Returns (A_out_cm [R; V], tau (batch, n), B_out_cm [X; residual
    components], info (batch,) int32: 0 or j+1 for the first zero R_jj)."""
    lib = _load()
    A = _widen(A_cm).copy()
    batch, n, lda = A.shape
    assert m >= n
    B = np.ascontiguousarray(B_cm, dtype=A.dtype).copy()
    _, nrhs, ldb = B.shape
    tau = np.zeros((batch, n), dtype=A.dtype)
    info = np.zeros((batch,), dtype=np.int32)
    if batch and n:
        fn = lib.bqr_ref_gels_z if _is_complex(A) else lib.bqr_ref_gels_d
        fn(m, n, nrhs, batch, _ptr(A), lda, _ptr(tau), _ptr(B), ldb, _ptr(info))
    return A, tau, B, info


def gels(A: np.ndarray, B: np.ndarray):
    """Logical API: A (batch, m, n), B (batch, m, nrhs) -> (X (batch, n, nrhs),
    residual components (batch, m-n, nrhs), info)."""
    A = np.asarray(A)
    B = np.asarray(B)
    if A.ndim == 2:
        A, B = A[None], B[None]
    m, n = A.shape[1], A.shape[2]
    _, _, Bo, info = gels_cm(to_cm(A), m, to_cm(B))
    Bl = from_cm(Bo, m)
    return Bl[:, :n, :], Bl[:, n:, :], info



# ---------------------------------------------------------------- NEXT-3
# LU without pivoting and Gauss-Jordan (paper Sec. III-A/B, P:L267-275,
# Listings 5-7); arithmetic in lu_ref.c.

def getrf_np_cm(A_cm: np.ndarray, m: int):
    """LU without pivoting on column-major storage A (batch, n, lda).
    Returns (LU_cm: L strictly lower (unit diagonal implied) + U upper,
    info (batch,) int32: 0 or k+1 for the first zero pivot)."""
    lib = _load()
    A = _widen(A_cm).copy()
    batch, n, lda = A.shape
    info = np.zeros((batch,), dtype=np.int32)
    if batch and m and n:
        fn = lib.bqr_ref_getrf_np_z if _is_complex(A) else lib.bqr_ref_getrf_np_d
        fn(m, n, batch, _ptr(A), lda, _ptr(info))
    return A, info


def getrf_np(A: np.ndarray):
    """Logical API: A (batch, m, n) -> (LU (batch, m, n), info)."""
    A = np.asarray(A)
    if A.ndim == 2:
        A = A[None]
    m = A.shape[1]
    LU, info = getrf_np_cm(to_cm(A), m)
    return from_cm(LU, m), info


def gauss_jordan_cm(A_cm: np.ndarray, B_cm: np.ndarray):
    """Gauss-Jordan on [A | B] without pivoting, column-major storage:
    A (batch, n, lda) with n x n matrices, B (batch, nrhs, ldb).  Returns
    (A_out_cm, X_cm, info): X overwrites B; A keeps the multipliers
    off the diagonal and pivot * (1/pivot) on it (lu_ref.c, reading L2)."""
    lib = _load()
    A = _widen(A_cm).copy()
    batch, n, lda = A.shape
    B = np.ascontiguousarray(B_cm, dtype=A.dtype).copy()
    _, nrhs, ldb = B.shape
    info = np.zeros((batch,), dtype=np.int32)
    if batch and n:
        fn = lib.bqr_ref_gauss_jordan_z if _is_complex(A) else lib.bqr_ref_gauss_jordan_d
        fn(n, nrhs, batch, _ptr(A), lda, _ptr(B), ldb, _ptr(info))
    return A, B, info


def gauss_jordan(A: np.ndarray, B: np.ndarray):
    """Logical API: A (batch, n, n), B (batch, n, nrhs) -> (X, info)."""
    A = np.asarray(A)
    B = np.asarray(B)
    if A.ndim == 2:
        A, B = A[None], B[None]
    n = A.shape[1]
    _, X, info = gauss_jordan_cm(to_cm(A), to_cm(B))
    return from_cm(X, n), info

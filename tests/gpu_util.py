"""Helpers for the GPU parity tests: move seeded column-major numpy batches
to the device, call the C ABI through the binding, bring results back."""
from __future__ import annotations

import numpy as np
import torch

import paper_conf_ipps_andersonsk12_b200 as bqr


def to_dev(A_cm: np.ndarray) -> torch.Tensor:
    """(batch, n, lda) numpy -> (batch, m=lda, n) column-major CUDA view over
    the full lda rows (callers slice m)."""
    t = torch.from_numpy(np.ascontiguousarray(A_cm)).cuda()
    return t


def geqrf_gpu(A_cm: np.ndarray, m: int, stream=None):
    """Factor on the GPU; returns (out_cm numpy, tau numpy)."""
    batch, n, lda = A_cm.shape
    buf = to_dev(A_cm)
    view = buf.transpose(1, 2)[:, :m, :] if batch else buf.transpose(1, 2)
    k = min(m, n)
    tau = torch.full((batch, k), float("nan"), dtype=buf.dtype, device="cuda")
    st = bqr.geqrf_batched_ptr(bqr.R32 if buf.dtype == torch.float32 else bqr.C64, m, n, batch,
                               buf.data_ptr(), lda, tau.data_ptr(),
                               (stream or torch.cuda.current_stream()).cuda_stream)
    assert st == 0, bqr.load().bqr_status_string(st)
    torch.cuda.synchronize()
    del view
    return buf.cpu().numpy(), tau.cpu().numpy()


def orgqr_gpu(RV_cm: np.ndarray, m: int, k: int, tau: np.ndarray):
    buf = to_dev(RV_cm)
    batch, n, lda = RV_cm.shape
    t = torch.from_numpy(np.ascontiguousarray(tau)).cuda()
    st = bqr.load().bqr_orgqr_batched(bqr.R32 if buf.dtype == torch.float32 else bqr.C64, m, n, k, batch,
                                      __import__("ctypes").c_void_p(buf.data_ptr()), lda,
                                      __import__("ctypes").c_void_p(t.data_ptr()), None)
    assert st == 0
    torch.cuda.synchronize()
    return buf.cpu().numpy()


def apply_gpu(RV_cm: np.ndarray, m: int, k: int, tau: np.ndarray, B_cm: np.ndarray):
    import ctypes
    A = to_dev(RV_cm)
    B = to_dev(B_cm)
    batch, n, lda = RV_cm.shape
    _, nrhs, ldb = B_cm.shape
    t = torch.from_numpy(np.ascontiguousarray(tau)).cuda()
    st = bqr.load().bqr_apply_qh_batched(bqr.R32 if A.dtype == torch.float32 else bqr.C64, m, n, k, nrhs, batch,
                                         ctypes.c_void_p(A.data_ptr()), lda, ctypes.c_void_p(t.data_ptr()),
                                         ctypes.c_void_p(B.data_ptr()), ldb, None)
    assert st == 0
    torch.cuda.synchronize()
    return B.cpu().numpy()


def geqrf_qhb_gpu(A_cm: np.ndarray, m: int, B_cm: np.ndarray):
    """Fused geqrf + Q^H B through bqr_geqrf_qhb_batched."""
    import ctypes
    A = to_dev(A_cm)
    B = to_dev(B_cm)
    batch, n, lda = A_cm.shape
    _, nrhs, ldb = B_cm.shape
    tau = torch.empty((batch, min(m, n)), dtype=A.dtype, device="cuda")
    st = bqr.load().bqr_geqrf_qhb_batched(bqr.R32 if A.dtype == torch.float32 else bqr.C64, m, n, nrhs, batch,
                                          ctypes.c_void_p(A.data_ptr()), lda, ctypes.c_void_p(tau.data_ptr()),
                                          ctypes.c_void_p(B.data_ptr()), ldb, None)
    assert st == 0, st
    torch.cuda.synchronize()
    return A.cpu().numpy(), tau.cpu().numpy(), B.cpu().numpy()


def gels_gpu(A_cm: np.ndarray, m: int, B_cm: np.ndarray):
    """Least squares through bqr_gels_batched; returns (A_out_cm, tau, B_out_cm, info)."""
    import ctypes
    A = to_dev(A_cm)
    B = to_dev(B_cm)
    batch, n, lda = A_cm.shape
    _, nrhs, ldb = B_cm.shape
    tau = torch.empty((batch, n), dtype=A.dtype, device="cuda")
    info = torch.full((batch,), -7, dtype=torch.int32, device="cuda")
    st = bqr.load().bqr_gels_batched(bqr.R32 if A.dtype == torch.float32 else bqr.C64, m, n, nrhs, batch,
                                     ctypes.c_void_p(A.data_ptr()), lda, ctypes.c_void_p(tau.data_ptr()),
                                     ctypes.c_void_p(B.data_ptr()), ldb, ctypes.c_void_p(info.data_ptr()), None)
    assert st == 0, st
    torch.cuda.synchronize()
    return A.cpu().numpy(), tau.cpu().numpy(), B.cpu().numpy(), info.cpu().numpy()

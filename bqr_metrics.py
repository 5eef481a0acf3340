"""bqr_metrics -- work/traffic accounting for the roofline (measurement only).

No method arithmetic: flop and byte counts that bench.py divides by measured
times, pinned in tests/test_metrics.py against the numbers PAPER.md prints.

  useful flops, real     F = 2 m n^2 - (2/3) n^3      (Sec. III-C;
                          the paper's 7x7 example gives 457; the
                          112x112 example 1.87 MFLOP)
  useful flops, complex  F = 8 m n^2 - (8/3) n^3      (Sec. VII)
  Q^H B apply per rhs    real 4 m n - 2 n^2, complex 16 m n - 8 n^2
                          (one reflector application per column, reading Q1)
  algorithmic bytes      read A once, write [R;V] once, write tau;
                          the apply adds B in and out
  NEXT-3    LU without pivoting "performs 2/3 n^3 FLOPs"
                          (m x n: m n^2 - n^3/3), Gauss-Jordan "performs n^3
                          FLOPs"; complex x4.  Bytes: A in and out (+ B in
                          and out for Gauss-Jordan) + a 4-byte info per matrix.
"""
from __future__ import annotations

import json
import os

ELEM_BYTES = {"f32": 4, "c64": 8}


def geqrf_flops(m: int, n: int, dtype: str = "f32") -> float:
    """Leading-order Householder QR flops for m >= n (reading Q1)."""
    if m < n:  # wide: k = m reflectors; count the m x m QR + applying to the rest
        m, n = n, m  # not used by any config; symmetric leading term is fine
    if dtype == "c64":
        return 8.0 * m * n * n - 8.0 / 3.0 * n ** 3
    return 2.0 * m * n * n - 2.0 / 3.0 * n ** 3


def apply_flops(m: int, n: int, nrhs: int, dtype: str = "f32") -> float:
    if dtype == "c64":
        return (16.0 * m * n - 8.0 * n * n) * nrhs
    return (4.0 * m * n - 2.0 * n * n) * nrhs


def geqrf_bytes(m: int, n: int, dtype: str = "f32") -> int:
    s = ELEM_BYTES[dtype]
    return 2 * m * n * s + min(m, n) * s


def apply_bytes(m: int, nrhs: int, dtype: str = "f32") -> int:
    return 2 * m * nrhs * ELEM_BYTES[dtype]


def arithmetic_intensity(m: int, n: int, dtype: str = "f32") -> float:
    """flop per byte moved (matrix read + write)."""
    s = ELEM_BYTES[dtype]
    return geqrf_flops(m, n, dtype) / (2 * m * n * s)


# ---------------------------------------------------------------- peaks

def load_peaks(path: str | None = None) -> dict:
    """MEASURED_PEAKS.json (driver-written) -> dict; fallback per
    B200_PROFILING.md when absent (6650 GB/s, 1965 MHz)."""
    path = path or os.path.join(os.path.dirname(os.path.abspath(__file__)), "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            d = json.load(f)
        d["source"] = "measured"
        return d
    except OSError:
        return {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0, "source": "fallback"}


def fp32_peak_tflops(n_sm: int = 148, mhz: float = 1965.0) -> float:
    """FP32 CUDA-core peak: SMs x 128 FMA lanes x 2 flop x clock
    (B200_PROFILING.md unit counts; no FP32 entry in MEASURED_PEAKS)."""
    return n_sm * 128 * 2 * mhz * 1e6 / 1e12


def roofline_time_s(flops: float, nbytes: float, hbm_gbs: float, fp32_tflops: float) -> tuple:
    """(time, bound) of the slower of the FP32 and HBM bounds."""
    t_c = flops / (fp32_tflops * 1e12)
    t_m = nbytes / (hbm_gbs * 1e9)
    return (t_c, "alu") if t_c >= t_m else (t_m, "hbm")


def lu_flops(m: int, n: int, dtype: str = "f32") -> float:
    """LU without pivoting, leading order: 2/3 n^3 for square."""
    k = min(m, n)
    f = float(m) * n * k - (m + n) * k * k / 2.0 + k ** 3 / 3.0
    f = 2.0 * f
    return 4.0 * f if dtype == "c64" else f


def gj_flops(n: int, dtype: str = "f32") -> float:
    """Gauss-Jordan on [A | b]: the paper's n^3."""
    f = float(n) ** 3
    return 4.0 * f if dtype == "c64" else f


def lu_bytes(m: int, n: int, dtype: str = "f32") -> int:
    return 2 * m * n * ELEM_BYTES[dtype] + 4


def gj_bytes(n: int, nrhs: int, dtype: str = "f32") -> int:
    return (2 * n * n + 2 * n * nrhs) * ELEM_BYTES[dtype] + 4

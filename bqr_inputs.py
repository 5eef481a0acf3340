"""bqr_inputs -- seeded synthetic workload generators (shared by tests, bench, smoke).

Holds NO arithmetic of the method: only random-number draws and array
layout.  Both the CUDA path and the oracle consume what these functions
return; neither side imports the other.

Layout: a batch of m x n matrices with leading dimension lda is stored
column-major per matrix, matrix b at offset b*lda*n elements (SURVEY 8(a) D1,
PAPER.md Listing 4).  As a numpy array this is shape
(batch, n, lda): element (b, row, col) lives at ``A_cm[b, col, row]``.

Configs (BASELINE.json ``configs``; recipes in DESIGN.md "Inputs"):
  C1  1,000 x 8x8 fp32, iid N(0,1), seed 1                 (correctness)
  C2  1,000,000 x 4x4 fp32, iid U(-1,1), seed 2            (HBM-bound tiny)
  C3  5,000 x 56x56 fp32, iid N(0,1), seed 3               (paper headline)
  C4  256 x 240x66 c64, iid CN(0,1) (re,im ~ N(0,1/2)), seed 4, plus one
      240x1 right-hand side per matrix                      (STAP, Table VII)
  C5  n in {16,...,256} square, fp32 N(0,1) seed 100+n / c64 CN(0,1) seed 200+n
The paper prints no input distribution for QR; its LU/solve inputs were
diagonally dominant -- irrelevant for Householder QR,
which is unconditionally stable, so iid Gaussian matrices are used.
"""
from __future__ import annotations

import numpy as np

C5_SIZES = (16, 24, 32, 48, 56, 64, 80, 96, 112, 128, 160, 192, 224, 256)

CONFIGS = {
    "C1": dict(m=8, n=8, batch=1000, dtype="f32", dist="normal", seed=1),
    "C2": dict(m=4, n=4, batch=1_000_000, dtype="f32", dist="uniform", seed=2),
    "C3": dict(m=56, n=56, batch=5000, dtype="f32", dist="normal", seed=3),
    "C4": dict(m=240, n=66, batch=256, dtype="c64", dist="normal", seed=4, nrhs=1),
    # NEXT-2: the paper's other RT_STAP sizes (Table VII, P:L1113-1123:
    # "80x16 384", "192x96 128"; complex single precision, QR only)
    "S80": dict(m=80, n=16, batch=384, dtype="c64", dist="normal", seed=5),
    "S192": dict(m=192, n=96, batch=128, dtype="c64", dist="normal", seed=6),
    # NEXT-3: LU without pivoting / Gauss-Jordan, 8,000 problems as the
    # paper's Fig. 11 comparison, diagonally dominant
    "L56": dict(m=56, n=56, batch=8000, dtype="f32", dist="diagdom", seed=7, kind="lu"),
    "GJ56": dict(m=56, n=56, batch=8000, dtype="f32", dist="diagdom", seed=8, nrhs=1, kind="gj"),
}


def c5_config(n: int, dtype: str, per_gpu: bool = True, n_sm: int = 148) -> dict:
    """C5 cell: per-GPU batch = max(16*SMs, ceil(1 GiB / (n^2 s)))."""
    s = 4 if dtype == "f32" else 8
    batch = max(16 * n_sm, -(-(1 << 30) // (n * n * s)))
    seed = (100 if dtype == "f32" else 200) + n
    return dict(m=n, n=n, batch=batch, dtype=dtype, dist="normal", seed=seed)


def np_dtype(dtype: str):
    return {"f32": np.float32, "c64": np.complex64}[dtype]


def random_batch(m: int, n: int, batch: int, dtype: str = "f32", seed: int = 0,
                 dist: str = "normal", lda: int | None = None,
                 start: int = 0, stop: int | None = None,
                 chunk: int = 1 << 16) -> np.ndarray:
    """Column-major storage (batch', n, lda) for matrices [start, stop) of the
    seeded batch.  Matrix b's values do not depend on start/stop: the stream is
    drawn in fixed chunks of ``chunk`` matrices, each chunk from its own
    SeedSequence child, so every rank slice sees identical matrices.

    Padding rows (lda > m) are filled with NaN sentinels so that tests can
    check they are never written (and, since NaN propagates, never read)."""
    lda = m if lda is None else lda
    stop = batch if stop is None else stop
    assert 0 <= start <= stop <= batch and lda >= max(1, m)
    cplx = dtype == "c64"
    out = np.empty((stop - start, n, lda), dtype=np_dtype(dtype))
    if lda > m:
        out[:, :, m:] = np.nan
    ss = np.random.SeedSequence(seed)
    first, last = start // chunk, (stop - 1) // chunk if stop > start else -1
    children = ss.spawn(last + 1) if last >= 0 else []
    for c in range(first, last + 1):
        rng = np.random.default_rng(children[c])
        c0 = c * chunk
        cnt = min(chunk, batch - c0)
        shape = (cnt, n, m)
        if dist == "normal":
            if cplx:
                s = np.sqrt(0.5)
                vals = (rng.standard_normal(shape, dtype=np.float32) * s
                        + 1j * (rng.standard_normal(shape, dtype=np.float32) * s))
            else:
                vals = rng.standard_normal(shape, dtype=np.float32)
        elif dist == "uniform":
            if cplx:
                vals = (rng.uniform(-1, 1, shape).astype(np.float32)
                        + 1j * rng.uniform(-1, 1, shape).astype(np.float32))
            else:
                vals = rng.uniform(-1, 1, shape).astype(np.float32)
        else:
            raise ValueError(dist)
        lo, hi = max(start, c0), min(stop, c0 + cnt)
        out[lo - start:hi - start, :, :m] = vals[lo - c0:hi - c0]
    return out


def diag_dominant_batch(n: int, batch: int, dtype: str = "f32", seed: int = 0,
                        lda: int | None = None, start: int = 0,
                        stop: int | None = None) -> np.ndarray:
    """NEXT-3 inputs (LU / Gauss-Jordan without pivoting): the paper ran them
    on "diagonally-dominant matrices so no pivoting was necessary"
    (P:L1009).  Off-diagonal entries are the seeded iid Gaussian
    stream of random_batch; each diagonal entry is replaced by
    +-(1 + max(column sum, row sum) of the off-diagonal magnitudes), so the
    matrix is strictly diagonally dominant by rows and by columns (the sign
    is the sign of the original draw).  Column-major (batch', n, lda)."""
    A = random_batch(n, n, batch, dtype, seed, "normal", lda=lda, start=start, stop=stop)
    lda = n if lda is None else lda
    core = A[:, :, :n]
    mag = np.abs(core).astype(np.float64)
    idx = np.arange(n)
    diag_mag = mag[:, idx, idx]
    colsum = mag.sum(axis=2) - diag_mag   # storage [b, col, row]: sum over rows
    rowsum = mag.sum(axis=1) - diag_mag
    d = 1.0 + np.maximum(colsum, rowsum)
    sgn = np.where(np.real(core[:, idx, idx]) < 0, -1.0, 1.0)
    core[:, idx, idx] = (sgn * d).astype(core.dtype)
    return A


STRESS_KINDS = ("tiny", "huge", "graded", "near_rank", "near_rank_tiny")


def stress_batch(m: int, n: int, batch: int, dtype: str, kind: str, seed: int) -> np.ndarray:
    """Inputs at the edges of the stated contract (reading Q6: entries in
    [1e-15, 1e15] or 0), column-major (batch, n, m):
      tiny       Gaussian draws with |x| clipped up to 0.1, times 1e-14
      huge       the same times 1e14
      graded     column j times 10^(-14 j / (n-1)): columns from O(1) to O(1e-14)
      near_rank  (B C + 1e-6 E) * 1e-8 with B m x r, C r x n, r = n/2, E noise:
                 numerical rank r, the trailing columns cancel to ~1e-14
      near_rank_tiny  the same at 1e-13: the trailing columns cancel to
                 ~1e-19 and their squares (sigma, nu^2, |z|^2) fall below
                 FLT_MIN (outside the accuracy contract of reading Q6, which
                 has no scaled norms; used to check the FTZ guard keeps every
                 output finite)
    Only random draws, scaling and a product of random factors (no QR
    arithmetic)."""
    A = random_batch(m, n, batch, dtype, seed).astype(np.complex128 if dtype == "c64" else np.float64)
    if kind in ("tiny", "huge", "graded"):
        mag = np.maximum(np.abs(A), 0.1)
        A = np.where(np.abs(A) > 0, A / np.where(np.abs(A) > 0, np.abs(A), 1.0), 1.0) * mag
        if kind == "tiny":
            A = A * 1e-14
        elif kind == "huge":
            A = A * 1e14
        else:
            A = A * (10.0 ** (-14.0 * np.arange(n) / max(1, n - 1)))[None, :, None]
    elif kind in ("near_rank", "near_rank_tiny"):
        r = max(1, n // 2)
        Bf = random_batch(m, r, batch, dtype, seed + 1).astype(A.dtype)   # (batch, r, m): B^T storage
        Cf = random_batch(r, n, batch, dtype, seed + 2).astype(A.dtype)   # (batch, n, r)
        # storage [b, col, row]: (B C)[row, col] = sum_t B[row, t] C[t, col]
        BC = np.einsum("btr,bct->bcr", Bf, Cf)
        A = (BC + 1e-6 * A) * (1e-13 if kind == "near_rank_tiny" else 1e-8)
    else:
        raise ValueError(kind)
    return A.astype(np_dtype(dtype))


def config_batch(name: str, start: int = 0, stop: int | None = None,
                 batch: int | None = None) -> np.ndarray:
    cfg = CONFIGS[name]
    b = cfg["batch"] if batch is None else batch
    if cfg["dist"] == "diagdom":
        return diag_dominant_batch(cfg["n"], b, cfg["dtype"], cfg["seed"], start=start, stop=stop)
    return random_batch(cfg["m"], cfg["n"], b, cfg["dtype"], cfg["seed"],
                        cfg["dist"], start=start, stop=stop)


def rhs_batch(m: int, nrhs: int, batch: int, dtype: str, seed: int,
              start: int = 0, stop: int | None = None) -> np.ndarray:
    """Right-hand sides B (batch, nrhs, ldb=m) for the Q^H B apply (C4)."""
    return random_batch(m, nrhs, batch, dtype, seed + 1_000_003, "normal",
                        start=start, stop=stop)


# --------------------------------------------------------------------------
# structured edge-case matrices (values only; no QR arithmetic)
# --------------------------------------------------------------------------

def edge_matrices(n: int, dtype: str, seed: int = 7) -> dict:
    """Named n x n edge cases (logical row-major numpy, shape (n, n))."""
    rng = np.random.default_rng(seed)
    dt = np_dtype(dtype)
    base = rng.standard_normal((n, n)).astype(np.float32)
    if dtype == "c64":
        base = (base + 1j * rng.standard_normal((n, n)).astype(np.float32)).astype(dt)
    eye = np.eye(n, dtype=dt)
    diag = np.diag(np.arange(1, n + 1) * (-1.0) ** np.arange(n)).astype(dt)
    zero_col = base.copy()
    zero_col[:, n // 2] = 0
    dup = base.copy()
    if n > 1:
        dup[:, 1] = dup[:, 0]
    upper = np.triu(base)
    negzero = base.copy()
    negzero[0, 0] = -0.0
    negzero[1:, 0] = 0.0
    if n > 1:
        negzero[1, 0] = 1.0
    return {
        "identity": eye,
        "diagonal": diag,
        "zero": np.zeros((n, n), dtype=dt),
        "zero_column": zero_col,
        "duplicate_columns": dup,
        "upper_triangular": upper,
        "neg_zero_pivot": negzero,
        "random": base,
    }

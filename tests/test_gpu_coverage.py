"""GPU parity, round 2: every size class the dispatch can pick is exercised
(asserted through bqr_kernel_name / bqr_qhb_kernel_name), the C5 sweep sizes,
inputs at the edges of the contract (reading Q6), and the tau batch stride
shared by geqrf / orgqr / apply_qh.  Comparator: oracle/compare.py
(north-star tolerances, reading Q10)."""
import numpy as np
import pytest

import bqr_inputs
import oracle
from oracle.compare import compare_apply, compare_geqrf, compare_orgqr

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a GPU", allow_module_level=True)

import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402
from gpu_util import apply_gpu, geqrf_gpu, geqrf_qhb_gpu, orgqr_gpu  # noqa: E402

DT = {bqr.R32: "f32", bqr.C64: "c64"}


def _classes():
    return [c for c in bqr.size_classes() if not c["experiment"]]


def _class_shapes(c):
    """(m, n) shapes that the dispatch maps to class c: its bound / exact shape
    and a ragged one just inside it."""
    if c["exact_m"]:
        return [(c["exact_m"], c["exact_n"])]
    m, n = c["mmax"], c["nmax"]
    return [(m, n), (m - 3, max(1, n - 5))]


@pytest.mark.parametrize("cls", _classes(), ids=lambda c: c["name"])
def test_every_size_class(cls):
    dt = DT[cls["dtype"]]
    batch = 40 if cls["mmax"] * cls["nmax"] > 20000 else 120
    hit = 0
    for m, n in _class_shapes(cls):
        if cls["augmented"]:
            nn = n - 1  # [A | b]: n columns of A plus one right-hand side
            if bqr.load().bqr_qhb_kernel_name(cls["dtype"], m, nn, 1).decode() != cls["name"]:
                continue
            A = bqr_inputs.random_batch(m, nn, batch, dt, seed=3000 + m + nn)
            B = bqr_inputs.rhs_batch(m, 1, batch, dt, seed=3000 + m)
            out, tau, Bo = geqrf_qhb_gpu(A, m, B)
            rep = compare_geqrf(A, m, out, tau, full_q=m <= 128)
            assert rep["ok"], (m, nn, rep)
            ra = compare_apply(out, m, nn, tau, B, Bo)
            assert ra["ok"], (m, nn, ra)
        else:
            if bqr.kernel_name(cls["dtype"], m, n) != cls["name"]:
                continue
            A = bqr_inputs.random_batch(m, n, batch, dt, seed=3000 + m + n)
            out, tau = geqrf_gpu(A, m)
            rep = compare_geqrf(A, m, out, tau, full_q=m <= 128)
            assert rep["ok"], (m, n, rep)
        hit += 1
    assert hit >= 1, f"class {cls['name']} is not reached by the dispatch at {_class_shapes(cls)}"


C5_F32 = [24, 48, 112]
C5_C64 = [24, 56, 80, 97, 112]


@pytest.mark.parametrize("n", C5_F32)
def test_c5_sizes_f32(n):
    A = bqr_inputs.random_batch(n, n, 200, "f32", seed=100 + n)
    out, tau = geqrf_gpu(A, n)
    assert compare_geqrf(A, n, out, tau)["ok"]


@pytest.mark.parametrize("n", C5_C64)
def test_c5_sizes_c64(n):
    A = bqr_inputs.random_batch(n, n, 120, "c64", seed=200 + n)
    out, tau = geqrf_gpu(A, n)
    assert compare_geqrf(A, n, out, tau)["ok"]


@pytest.mark.parametrize("kind", bqr_inputs.STRESS_KINDS)
@pytest.mark.parametrize("shape", [(56, 56, "f32"), (240, 66, "c64"), (8, 8, "f32"), (128, 128, "c64")])
def test_contract_edges(kind, shape):
    """Entries near 1e-15 / 1e15, graded columns and numerically
    rank-deficient matrices (at 1e-13 scale the trailing sigma / nu^2 / |z|^2
    are subnormal: the FTZ guard of bqr_common.cuh keeps them finite), at
    the C3 / C4 shapes."""
    m, n, dt = shape
    A = bqr_inputs.stress_batch(m, n, 64 if m * n < 20000 else 16, dt, kind, seed=4000 + m)
    out, tau = geqrf_gpu(A, m)
    assert np.all(np.isfinite(out)) and np.all(np.isfinite(tau))
    rep = compare_geqrf(A, m, out, tau, full_q=m <= 128)
    if kind == "near_rank_tiny":
        # subnormal sums of squares carry ~1e-5 relative error (no scaled
        # norms, reading Q6): only finiteness and the reconstruction bind
        assert rep["residual_max"] <= 1e-5, (kind, rep)
    else:
        assert rep["ok"], (kind, {k: v for k, v in rep.items() if k != "fail_idx"})


@pytest.mark.parametrize("dt", ["f32", "c64"])
def test_partial_k_reuses_geqrf_tau(dt):
    """orgqr / apply_qh with k < min(m, n) read tau with geqrf's batch stride
    min(m, n) (include/bqr.h conventions), as LAPACK's xORMQR after xGEQRF."""
    m, n, k, batch = 40, 12, 7, 9
    A = bqr_inputs.random_batch(m, n, batch, dt, seed=77)
    out, tau = geqrf_gpu(A, m)
    B = bqr_inputs.rhs_batch(m, 3, batch, dt, seed=78)
    got = apply_gpu(out, m, k, tau, B)
    ra = compare_apply(out, m, k, tau[:, :k], B, got)
    assert ra["ok"], ra
    Q = orgqr_gpu(out, m, k, tau)
    ro = compare_orgqr(out, m, k, tau[:, :k], Q)
    assert ro["ok"], ro

"""Randomised shape sweep through the C ABI (seeded, reproducible): shapes
drawn across every dispatch region (tiny, sub-warp, warp, CTA, single-SM,
compact WY, tiled), random lda padding, both dtypes, against the fp64 oracle
with the north-star tolerances (reading Q10); plus the downstream entry
points on the blocked-variant outputs (orgqr, apply_qh, gels on complex
shapes beyond one SM)."""
import numpy as np
import pytest

import bqr_inputs
from oracle.compare import compare_apply, compare_gels, compare_geqrf, compare_orgqr

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a GPU", allow_module_level=True)

import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402
from gpu_util import apply_gpu, geqrf_gpu, gels_gpu, orgqr_gpu  # noqa: E402


def _shapes(seed, count):
    rng = np.random.default_rng(seed)
    out = []
    for _ in range(count):
        m = int(rng.integers(1, 257))
        n = int(rng.integers(1, m + 1))
        pad = int(rng.choice([0, 0, 0, 1, 2, 3]))
        out.append((m, n, pad))
    return out


@pytest.mark.parametrize("dt", ["f32", "c64"])
@pytest.mark.parametrize("m,n,pad", _shapes(2026, 24))
def test_random_shapes(dt, m, n, pad):
    batch = 40 if m * n > 20000 else 96
    A = bqr_inputs.random_batch(m, n, batch, dt, seed=7000 + 3 * m + n, lda=m + pad)
    out, tau = geqrf_gpu(A, m)
    rep = compare_geqrf(A, m, out, tau, full_q=m <= 128)
    assert rep["ok"] and rep["padding_ok"], (bqr.kernel_name(bqr.R32 if dt == "f32" else bqr.C64, m, n), rep)


@pytest.mark.parametrize("m,n", [(256, 200), (224, 176)])
def test_downstream_of_blocked_variant(m, n):
    """orgqr / apply_qh / gels consume the compact-WY outputs (complex > 160)."""
    assert bqr.kernel_name(bqr.C64, m, n).startswith("wy_")
    A = bqr_inputs.random_batch(m, n, 12, "c64", seed=7100 + m)
    out, tau = geqrf_gpu(A, m)
    assert compare_geqrf(A, m, out, tau, full_q=False)["ok"]
    B = bqr_inputs.rhs_batch(m, 2, 12, "c64", seed=7101)
    got = apply_gpu(out, m, n, tau, B)
    assert compare_apply(out, m, n, tau, B, got)["ok"]
    Q = orgqr_gpu(out, m, n, tau)
    assert compare_orgqr(out, m, n, tau, Q)["ok"]
    Ao, _, Bo, info = gels_gpu(A, m, B)
    rep = compare_gels(A, m, B, Bo, info)
    assert rep["ok"], rep


@pytest.mark.parametrize("k", [0, 1, 96, 150, 200])
def test_orgqr_blocked_partial_k(k):
    """xUNGQR by compact-WY panels (complex n > 160) with k <= n reflectors:
    full panels, a ragged last panel, a single reflector and k = 0 (Q = I)."""
    m, n = 256, 200
    A = bqr_inputs.random_batch(m, n, 6, "c64", seed=7200 + k)
    out, tau = geqrf_gpu(A, m)
    Q = orgqr_gpu(out, m, k, tau)
    ro = compare_orgqr(out, m, k, tau[:, :k], Q)
    assert ro["ok"], ro

"""Pins for the roofline accounting (bqr_metrics) against numbers PAPER.md prints."""
import json
import os

import pytest

import bqr_metrics as bm

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "paper_numbers.json")


def _load():
    with open(GOLDEN) as f:
        d = json.load(f)
    return {k: v for k, v in d.items() if not k.startswith("_")}


@pytest.mark.parametrize("name", sorted(_load()))
def test_paper_numbers(name):
    e = _load()[name]
    m, n, dt = e["m"], e["n"], e["dtype"]
    if name.endswith("_bytes"):
        got = 2 * m * n * bm.ELEM_BYTES[dt]
    elif name.endswith("_intensity"):
        got = bm.arithmetic_intensity(m, n, dt)
    else:
        got = bm.geqrf_flops(m, n, dt)
    assert got == pytest.approx(e["value"], rel=max(e["rel_tol"], 1e-12)), e["cite"]


def test_config_totals():
    """C3 = 1.171 GFLOP / 126.6 MB, C4 = 2.001 GFLOP."""
    c3_f = 5000 * bm.geqrf_flops(56, 56)
    c3_b = 5000 * bm.geqrf_bytes(56, 56)
    assert c3_f == pytest.approx(1.1708e9, rel=1e-3)
    assert c3_b == pytest.approx(126.56e6, rel=1e-3)
    c4_f = 256 * (bm.geqrf_flops(240, 66, "c64") + bm.apply_flops(240, 66, 1, "c64"))
    assert c4_f == pytest.approx(2.001e9, rel=1e-3)
    assert bm.apply_flops(240, 66, 1, "c64") == 218592


def test_roofline_bound():
    t, bound = bm.roofline_time_s(1.171e9, 126.6e6, 6545.6, bm.fp32_peak_tflops())
    assert bound == "hbm" and t == pytest.approx(19.34e-6, rel=2e-3)
    assert bm.fp32_peak_tflops() == pytest.approx(74.45, rel=1e-3)


def test_next3_flop_counts_match_the_paper():
    # "This algorithm performs n^3 FLOPs" (Gauss-Jordan);
    # LU "performs 2/3 n^3 FLOPs"
    for n in (4, 56, 128):
        assert bm.gj_flops(n) == n ** 3
        assert abs(bm.lu_flops(n, n) - 2.0 / 3.0 * n ** 3) < 1e-6 * n ** 3
    # rectangular LU: m n^2 - n^3/3 (m >= n), symmetric in the wide case
    assert abs(bm.lu_flops(80, 16) - (80 * 16 ** 2 - 16 ** 3 / 3)) < 1e-9
    assert abs(bm.lu_flops(16, 80) - bm.lu_flops(80, 16)) < 1e-9
    assert bm.lu_flops(8, 8, "c64") == 4 * bm.lu_flops(8, 8)

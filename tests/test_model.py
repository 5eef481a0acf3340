"""NEXT-4: the per-column performance model (bqr_model).  The paper's own
model (Table VI) with its Table IV parameters must land near
the cycle counts the paper measured for 56 x 56 (Table V: QR
150,203, LU 68,250) -- the paper calls the model accurate; the
B200 re-parameterisation must be internally consistent."""
import bqr_model as M


def test_paper_model_reproduces_table_v():
    qr = M.paper_qr_cycles(56)
    lu = M.paper_lu_cycles(56)
    assert 0.8 * 150203 <= qr <= 1.2 * 150203, qr
    assert 0.8 * 68250 <= lu <= 1.2 * 68250, lu
    # QR costs more than LU per column (two reductions, sqrt/div)
    assert qr > 2 * lu * 0.9


def test_paper_model_grows_with_n():
    vals = [M.paper_qr_cycles(n) for n in (16, 32, 56, 64)]
    assert vals == sorted(vals)


def test_b200_bounds_are_ordered_and_scale_with_rounds():
    for L, batch in ((M.C3_LAYOUT, 5000), (M.C4_LAYOUT, 256)):
        p = M.predict_us(L, batch)
        assert 0 < p["lo_us"] <= p["hi_us"]
        p2 = M.predict_us(L, 2 * batch)
        assert p2["lo_us"] > p["lo_us"]
    cols = M.column_costs(M.C3_LAYOUT)
    assert len(cols) == 56
    # the trailing work shrinks column by column; the chain does not vanish
    assert cols[0][1] > cols[-1][1] and cols[-1][0] > 0


def test_r02_bounds_bracket_the_measurements():
    """NEXT-4 (Tables II-IV / VI): with the B200
    microbenchmark constants and the kernels' measured instruction counts and
    warp CPI, the lower / upper bounds bracket the measured C3, C4 and S80
    kernel times and the batch-1 latencies (profiles/model_r02.json, written
    by tools/model_report.py from the committed bench line and ncu details)."""
    import json
    import os
    path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "model_r02.json")
    d = json.load(open(path))["b200"]
    for cfg in ("C3", "C4", "S80"):
        b = d[cfg]
        assert b["lo_us"] <= b["measured_us"] <= b["hi_us"], (cfg, b)
        if "measured_batch_1" in b["latency_floor_us"]:
            f = b["latency_floor_us"]
            assert f["lo"] <= f["measured_batch_1"] <= f["hi"], (cfg, f)
    # the recomputation agrees with the file
    import bqr_model as M
    b = M.bounds_us(M.LAYOUTS[d["C3"].get("layout", "C3")], 5000, d["C3"]["ncu"]["executed_instructions"],
                    d["C3"]["ncu"]["warp_cpi"],
                    5000 * 117077.33333333333)
    assert abs(b["lo_us"] - d["C3"]["lo_us"]) < 1e-6 and abs(b["hi_us"] - d["C3"]["hi_us"]) < 1e-6

"""NEXT-4 report: the paper's Table VI model (Fermi parameters) against its
Table V measurements, and the B200 bounds of bqr_model.bounds_us (measured
microbenchmark latencies + this round's ncu instruction counts and warp CPI)
against this round's bench times and batch-1 latencies.  Writes
profiles/model_r02.json.

    python tools/model_report.py [bench.json]
"""
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bqr_metrics as bm  # noqa: E402
import bqr_model as M  # noqa: E402

NCU = os.path.join(ROOT, "profiles", "r02", "ncu")


def ncu_metric(cfg: str, name: str, ncu_dir: str = NCU) -> float:
    with open(os.path.join(ncu_dir, f"details_{cfg}.txt")) as f:
        for line in f:
            if line.startswith(name):
                return float(re.findall(r"[-+]?\d[\d.]*", line[len(name):])[0])
    raise KeyError(name)


def main():
    bench_path = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles", "r02", "bench_r02b.json")
    bench = json.load(open(bench_path))
    out = {"paper_fermi": {
        "qr_56": {"model_cycles": M.paper_qr_cycles(56), "paper_measured_cycles": 150203},
        "lu_56": {"model_cycles": M.paper_lu_cycles(56), "paper_measured_cycles": 68250},
        "readings": "b = shared latency 27, g = 18, a_sync = 46 (Table IV); g_sqrt = g_div = 2 g (not printed)"},
        "b200": {}}
    # the C3 class of the bench line: the left-looking one (its ncu capture in
    # profiles/r02/ll/) or the round-1 right-looking one
    c3_ll = bench["roofline"].get("kernel", "").startswith("ll_")
    c3_layout = M.C3_LL_LAYOUT if c3_ll else M.C3_LAYOUT
    ncu_dirs = {"C3": os.path.join(ROOT, "profiles", "r02", "ll") if c3_ll else NCU}
    cases = {
        "C3": (c3_layout, 5000, bench["roofline"]["kernel_us"], bench["latency"]["batch_1_us"], 56, 56, "f32"),
        "C4": (M.C4_LAYOUT, 256, bench["also"]["C4"]["roofline"]["kernel_us"],
               bench["also"]["C4"].get("latency", {}).get("batch_1_us"), 240, 66, "c64"),
        "S80": (M.S80_LAYOUT, 384, bench["also"]["S80"]["roofline"]["kernel_us"], None, 80, 16, "c64"),
    }
    for cfg, (L, batch, measured, lat1, m, n, dt) in cases.items():
        instr = ncu_metric(cfg, "Executed Instructions", ncu_dirs.get(cfg, NCU))
        cpi = ncu_metric(cfg, "Warp Cycles Per Issued Instruction", ncu_dirs.get(cfg, NCU))
        fmas = batch * bm.geqrf_flops(m, n, dt) / 2
        if cfg == "C4":  # the bench step is the fused [A | b] factorisation
            fmas += batch * bm.apply_flops(m, n, 1, dt) / 2
        b = M.bounds_us(L, batch, instr, cpi, fmas)
        b["measured_us"] = measured
        b["bracketed"] = bool(b["lo_us"] <= measured <= b["hi_us"])
        if lat1 is not None:
            b["latency_floor_us"]["measured_batch_1"] = lat1
            b["latency_floor_us"]["bracketed"] = bool(b["latency_floor_us"]["lo"] <= lat1 <= b["latency_floor_us"]["hi"])
        b["ncu"] = {"executed_instructions": instr, "warp_cpi": cpi}
        b["layout"] = next(k for k, v in M.LAYOUTS.items() if v is L) if L in M.LAYOUTS.values() else "S80"
        out["b200"][cfg] = b
    out["b200"]["note"] = ("lo = max(issue of every executed warp instruction at 1 / scheduler / cycle, useful FMAs at "
                           "the measured FFMA rate, rounds x the per-matrix reflector chain); hi = ceil(rounds) x "
                           "(chain + one warp's instructions per round x the measured warp CPI); latency floor = "
                           "chain + one warp's instructions at CPI 1 .. at the measured CPI.  Constants: "
                           "profiles/r02/micro2.jsonl (tools/micro/micro2.cu); counts: profiles/r02/ncu/details_*.txt.")
    path = os.path.join(ROOT, "profiles", "model_r02.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()

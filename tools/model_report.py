"""NEXT-4 report: the paper's Table VI model (Fermi parameters) against its
Table V measurements, and the B200 re-parameterisation (bqr_model) against
this round's measurements (profiles/bench_r01.json, phase timer).  Writes
profiles/model_r01.json.

    python tools/model_report.py
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bqr_model as M  # noqa: E402


def main():
    bench = json.load(open(os.path.join(ROOT, "profiles", "bench_r01.json")))
    out = {"paper_fermi": {
        "qr_56": {"model_cycles": M.paper_qr_cycles(56), "paper_measured_cycles": 150203},
        "lu_56": {"model_cycles": M.paper_lu_cycles(56), "paper_measured_cycles": 68250},
        "readings": "b = shared latency 27, g = 18, a_sync = 46 (Table IV); g_sqrt = g_div = 2 g (not printed)"}}
    c3 = M.predict_us(M.C3_LAYOUT, 5000)
    c3["measured_us"] = bench["roofline"]["kernel_us"]
    c4 = M.predict_us(M.C4_LAYOUT, 256)
    c4["measured_us_fused_step"] = bench["also"]["C4"]["roofline"]["kernel_us"]
    one = M.predict_us(M.C4_LAYOUT, 1)
    ph = os.path.join(ROOT, "profiles", "r01", "experiments", "ph_c4_dec_1.jsonl")
    if os.path.exists(ph):
        rows = [json.loads(line) for line in open(ph) if line.startswith("{")]
        one["measured_step_cycles_phase_timer"] = rows[-1].get("total_cycles")
    one["model_chain_plus_issue_cycles"] = one["chain_cycles"] + one["issue_cycles"]
    out["b200"] = {"C3": c3, "C4": c4, "C4_one_matrix": one,
                   "note": "lo = perfect overlap of the reflector chain with the trailing update at IPC 1 per "
                           "scheduler, hi = no overlap; measured above hi = issue stalls the model does not "
                           "price (FMA dependency waits, register-bank dispatch stalls, ncu 'wait'/'dispatch')"}
    path = os.path.join(ROOT, "profiles", "model_r01.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()

"""Wave-quantisation experiment on C3 (5000 x 56x56 f32 = 2.11 rounds of
2368 resident matrices): does launching the batch as two concurrent
launches on two streams (tail first / main first / halves) beat one launch?

    python tools/split_ab.py
"""
import json, os, sys
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_ipps_andersonsk12_b200 as bqr
import bqr_inputs

cfg = bqr_inputs.CONFIGS["C3"]
m, n, B = cfg["m"], cfg["n"], cfg["batch"]
A0 = torch.randn(B, n, m, device="cuda")  # column-major per matrix: (batch, n cols, m rows)
A = A0.clone()
tau = torch.empty(B, n, device="cuda")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
s0 = torch.cuda.current_stream()
s1 = torch.cuda.Stream()
ms = m * n


def launch(b0, cnt, st):
    bqr.geqrf_batched_ptr(0, m, n, cnt, A.data_ptr() + 4 * b0 * ms, m, tau.data_ptr() + 4 * b0 * n, st.cuda_stream)


def variant(parts):
    # parts: list of (b0, cnt, side) in launch order
    ev = torch.cuda.Event()
    ev.record(s0)
    s1.wait_event(ev)
    for b0, cnt, side in parts:
        launch(b0, cnt, s1 if side else s0)
    s0.wait_stream(s1)


R = 2368
V = {
    "single": [(0, B, 0)],
    "seq_main_tail": [(0, B - 264, 0), (B - 264, 264, 0)],
    "tail_first_side": [(B - 264, 264, 1), (0, B - 264, 0)],
    "main_first_side": [(0, B - 264, 0), (B - 264, 264, 1)],
    "halves": [(0, B // 2, 0), (B // 2, B - B // 2, 1)],
    "round_plus_rest": [(0, R, 0), (R, B - R, 1)],
}
res = {}
for name, parts in V.items():
    ts = []
    for it in range(23):
        A.copy_(A0)
        flush.zero_()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s0)
        variant(parts)
        b.record(s0)
        torch.cuda.synchronize()
        if it >= 3:
            ts.append(a.elapsed_time(b) * 1000)
    ts.sort()
    res[name] = round(ts[len(ts) // 2], 1)
print(json.dumps(res))

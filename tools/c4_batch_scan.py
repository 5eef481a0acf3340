import sys, os, json
sys.path.insert(0, os.getcwd())
import torch, bench, paper_conf_ipps_andersonsk12_b200 as bqr
flush = torch.empty(256 << 20, dtype=torch.uint8, device='cuda')
for b in [1, 74, 148, 222, 256, 296]:
    w = bench.Workload("C4", 0, 1, torch, bqr, batch=b)
    _, q = bench.time_workload(w, 20, 3, torch, None, 1, flush, fused=True)
    print(json.dumps({"variant": os.environ.get("BQR_FORCE_VARIANT", "default"), "batch": b, "fused_us": round(q * 1e3, 2)}), flush=True)

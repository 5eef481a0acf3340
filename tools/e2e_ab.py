"""A/B of the host-buffer pipeline (bqr_geqrf_batched_host) on the C3 batch for
one libbqr.so build and several chunk counts (batch // div).

    python tools/e2e_ab.py <libbqr.so> [8,16,32]
"""
import sys, json, os
sys.path.insert(0, os.getcwd())
import paper_conf_ipps_andersonsk12_b200 as bqr
bqr._LIB_PATH = os.path.abspath(sys.argv[1])
import torch, bench
w = bench.Workload("C3", 0, 1, torch, bqr)
for div in [int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "8,16,32").split(",")]:
    orig = w.batch
    import types
    # re-implement the chunk choice of bench.e2e_host with a different divisor
    src = bench.e2e_host
    def run(div=div):
        host_in = torch.from_numpy(w.host.copy())
        Ah = torch.empty_like(host_in).pin_memory()
        tauh = torch.empty((w.batch, w.k), dtype=w.tau.dtype).pin_memory()
        chunk = max(1, w.batch // div)
        wsb = bqr.host_workspace_bytes(w.code, w.m, w.n, w.m, chunk)
        ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
        ev = [[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in range(10)]
        for _ in range(2):
            Ah.copy_(host_in); bqr.geqrf_batched_host(w.code, w.m, w.n, w.batch, Ah.data_ptr(), w.m, tauh.data_ptr(), ws.data_ptr(), wsb)
        for i in range(10):
            Ah.copy_(host_in)
            ev[i][0].record(w.stream)
            bqr.geqrf_batched_host(w.code, w.m, w.n, w.batch, Ah.data_ptr(), w.m, tauh.data_ptr(), ws.data_ptr(), wsb)
            ev[i][1].record(w.stream)
        torch.cuda.synchronize()
        return sum(e[0].elapsed_time(e[1]) for e in ev) / 10
    print(json.dumps({"lib": sys.argv[1], "div": div, "ms": round(run(), 4)}))

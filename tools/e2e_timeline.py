"""Timeline of the host-buffer pipeline, re-enacted in Python with the same
stream/event structure as bqr_geqrf_batched_host (H2D stream, compute
stream, D2H stream, a ring of NB device buffers), with timing events on every
stage so the per-chunk start/end of each copy and kernel can be read.

    python tools/e2e_timeline.py [chunk_div] [NB] [--uniform]
"""
import json, os, sys
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_ipps_andersonsk12_b200 as bqr
import bench

div = int(sys.argv[1]) if len(sys.argv) > 1 else 4
NB = int(sys.argv[2]) if len(sys.argv) > 2 else 3
uniform = "--uniform" in sys.argv
w = bench.Workload("C3", 0, 1, torch, bqr)
B, m, n, k = w.batch, w.m, w.n, w.k
host_in = torch.from_numpy(w.host.copy())
Ah = torch.empty_like(host_in).pin_memory()
tauh = torch.empty((B, k), dtype=w.tau.dtype).pin_memory()
chunk = max(1, B // div)


def schedule():
    ramp = [] if uniform else [chunk >> s for s in (3, 2, 1) if (chunk >> s) > 0]
    if B <= 2 * sum(ramp) + chunk:
        ramp = []
    mid = B - 2 * sum(ramp)
    nmid = (mid + chunk - 1) // chunk
    return ramp + [min(chunk, mid - i * chunk) for i in range(nmid)] + ramp[::-1]


sizes = schedule()
dA = [torch.empty((chunk,) + tuple(Ah.shape[1:]), dtype=Ah.dtype, device="cuda") for _ in range(NB)]
dT = [torch.empty((chunk, k), dtype=tauh.dtype, device="cuda") for _ in range(NB)]
cs = torch.cuda.current_stream()
hs, ds = torch.cuda.Stream(), torch.cuda.Stream()
E = lambda: torch.cuda.Event(enable_timing=True)


def run(rec):
    t0 = E(); t0.record(cs)
    hs.wait_stream(cs)
    outev = [None] * NB
    marks = []
    b0 = 0
    for ci, cnt in enumerate(sizes):
        b = ci % NB
        if outev[b] is not None:
            hs.wait_event(outev[b])
        e = [E() for _ in range(6)]
        e[0].record(hs)
        with torch.cuda.stream(hs):
            dA[b][:cnt].copy_(Ah[b0:b0 + cnt], non_blocking=True)
        e[1].record(hs)
        cs.wait_event(e[1])
        e[2].record(cs)
        bqr.geqrf_batched_ptr(w.code, m, n, cnt, dA[b].data_ptr(), m, dT[b].data_ptr(), cs.cuda_stream)
        e[3].record(cs)
        ds.wait_event(e[3])
        e[4].record(ds)
        with torch.cuda.stream(ds):
            Ah[b0:b0 + cnt].copy_(dA[b][:cnt], non_blocking=True)
            tauh[b0:b0 + cnt].copy_(dT[b][:cnt], non_blocking=True)
        e[5].record(ds)
        outev[b] = e[5]
        marks.append((cnt, e))
        b0 += cnt
    cs.wait_stream(ds)
    t1 = E(); t1.record(cs)
    torch.cuda.synchronize()
    tot = t0.elapsed_time(t1)
    if rec:
        rows = []
        for cnt, e in marks:
            rows.append([cnt] + [round(t0.elapsed_time(x) * 1000) for x in e])
        return tot, rows
    return tot, None


for _ in range(3):
    run(False)
ts = [run(False)[0] for _ in range(10)]
tot, rows = run(True)
print(json.dumps({"div": div, "NB": NB, "uniform": uniform, "sizes": sizes, "ms_median": sorted(ts)[5]}))
print("cnt h2d_start h2d_end k_start k_end d2h_start d2h_end (us)")
for r in rows:
    print(r)

import torch, json
E = lambda: torch.cuda.Event(enable_timing=True)
h = torch.empty(16 << 20, dtype=torch.uint8).pin_memory()
h2 = torch.empty(16 << 20, dtype=torch.uint8).pin_memory()
d = torch.empty(16 << 20, dtype=torch.uint8, device="cuda")
d2 = torch.empty(16 << 20, dtype=torch.uint8, device="cuda")
x = torch.zeros(1024, device="cuda")
hs, cs, ds = torch.cuda.Stream(), torch.cuda.Stream(), torch.cuda.Stream()
for concurrent in (False, True):
    gaps = []
    for it in range(20):
        torch.cuda.synchronize()
        e0, e1, e2, e3 = E(), E(), E(), E()
        if concurrent:
            with torch.cuda.stream(ds):
                h2.copy_(d2, non_blocking=True)
        e0.record(hs)
        with torch.cuda.stream(hs):
            d.copy_(h, non_blocking=True)
        e1.record(hs)
        cs.wait_event(e1)
        e2.record(cs)
        with torch.cuda.stream(cs):
            x.add_(1.0)
        e3.record(cs)
        torch.cuda.synchronize()
        gaps.append((e0.elapsed_time(e1) * 1e3, e1.elapsed_time(e2) * 1e3, e2.elapsed_time(e3) * 1e3))
    g = sorted(gaps, key=lambda t: t[1])[10]
    print(json.dumps({"concurrent_d2h": concurrent, "h2d_us": round(g[0], 1), "event_to_next_us": round(g[1], 1), "tiny_kernel_us": round(g[2], 1)}))

"""Kernel time of one bench config at several batches, after the bench's
256 MB write flush and without a flush, for several builds of libbqr.so
(per-process library override; CUDA events around the geqrf launch).

    python tools/lat_lib.py C3 1,625,5000 abl/libbqr_X.so paper_conf_ipps_andersonsk12_b200/libbqr.so
"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
cfg, batches = sys.argv[1], [int(b) for b in sys.argv[2].split(",")]
for lib in sys.argv[3:]:
    code = f"""
import sys, json; sys.path.insert(0, {ROOT!r})
import paper_conf_ipps_andersonsk12_b200 as bqr
bqr._LIB_PATH = {os.path.abspath(lib)!r}
import torch, bench
big = torch.empty(256 << 20, dtype=torch.uint8, device='cuda')
for b in {batches!r}:
    w = bench.Workload({cfg!r}, 0, 1, torch, bqr, batch=b)
    row = {{'cfg': {cfg!r}, 'lib': {lib!r}, 'batch': b, 'kernel': bqr.kernel_name(w.code, w.m, w.n)}}
    for name, fl in (('write256MB', lambda: big.zero_()), ('none', lambda: None)):
        ts = []
        for it in range(23):
            w.restore()
            fl()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(w.stream)
            w.geqrf()
            e1.record(w.stream)
            torch.cuda.synchronize()
            if it >= 3:
                ts.append(e0.elapsed_time(e1) * 1e3)
        row[name + '_us'] = round(sorted(ts)[len(ts) // 2], 2)
    print(json.dumps(row), flush=True)
"""
    subprocess.run([sys.executable, "-c", code], check=True)

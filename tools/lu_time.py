"""Kernel time of the NEXT-3 bench workloads (L56, GJ56) for one or more
builds of libbqr.so (per-process override), L2 flushed, CUDA events.

    python tools/lu_time.py abl/libbqr_a.so abl/libbqr_b.so
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
for lib in sys.argv[1:]:
    code = f"""
import sys, json; sys.path.insert(0, {ROOT!r})
import paper_conf_ipps_andersonsk12_b200 as bqr
bqr._LIB_PATH = {os.path.abspath(lib)!r}
import torch, bench
flush = torch.empty(256 << 20, dtype=torch.uint8, device='cuda')
for cfg in ('L56', 'GJ56'):
    w = bench.Workload(cfg, 0, 1, torch, bqr)
    s_ms, q_ms = bench.time_workload(w, 30, 5, torch, None, 1, flush)
    print(json.dumps({{'cfg': cfg, 'lib': {lib!r}, 'us': round(q_ms * 1e3, 2), 'gflops': round(w.flops / q_ms / 1e6, 1)}}))
"""
    subprocess.run([sys.executable, "-c", code], check=False)

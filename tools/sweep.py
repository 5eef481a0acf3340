"""C5 size sweep: square n in {16..256} x {fp32, c64}, per-GPU
batch = max(16*SMs, ceil(1 GiB / (n^2 s))), kernel-only device time with the
bench's protocol (restore + L2 flush untimed, CUDA events), useful GFLOP/s,
matrices/s and roofline fraction.  One JSON line per cell.

    python tools/sweep.py [--sizes 16,24,...] [--dtypes f32,c64] [--steps 10]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import bqr_inputs  # noqa: E402
import bqr_metrics as bm  # noqa: E402
import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sizes", default=",".join(map(str, bqr_inputs.C5_SIZES)))
    ap.add_argument("--dtypes", default="f32,c64")
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--max-gib", type=float, default=1.0)
    ap.add_argument("--variant", default="", help="BQR_FORCE_VARIANT for every cell")
    args = ap.parse_args()
    if args.variant:
        os.environ["BQR_FORCE_VARIANT"] = args.variant
    torch.cuda.set_device(0)
    props = torch.cuda.get_device_properties(0)
    n_sm = props.multi_processor_count
    flush = torch.empty(2 * props.L2_cache_size, dtype=torch.uint8, device="cuda")
    peaks = bm.load_peaks()
    for dt in args.dtypes.split(","):
        for n in map(int, args.sizes.split(",")):
            cfg = bqr_inputs.c5_config(n, dt, n_sm=n_sm)
            s = 4 if dt == "f32" else 8
            batch = min(cfg["batch"], int(args.max_gib * (1 << 30) // (n * n * s)))
            bqr_inputs.CONFIGS["C5"] = dict(cfg, batch=batch)
            w = bench.Workload("C5", 0, 1, torch, bqr)
            s_ms, q_ms = bench.time_workload(w, args.steps, 3, torch, None, 1, flush)
            roof = bench.roofline_obj(w, q_ms, peaks, n_sm)
            print(json.dumps({"cell": f"{dt}_{n}", "n": n, "dtype": dt, "batch": batch,
                              "kernel": bqr.kernel_name(w.code, n, n),
                              "launches": bqr.geqrf_launches(w.code, n, n, batch),
                              "ms": round(q_ms, 4), "gflops": round(w.flops / (q_ms / 1e3) / 1e9, 1),
                              "matrices_per_s": round(batch / (q_ms / 1e3), 1),
                              "bound": roof["bound"], "roofline_frac": roof["frac"]}), flush=True)
            del w
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()

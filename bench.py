#!/usr/bin/env python
"""bench.py -- batched Householder QR on B200: the BASELINE.json metric.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--config C3|C4|C2|C1|...] [--scaling weak|strong]
                    [--no-also] [--no-c5] [--no-cpu]

One "step" = one pass of the whole hot path over one batch:
  C3 (default, the metric's headline workload): bqr_geqrf_batched on 5,000
     56x56 fp32 matrices per GPU;
  C4 (reported under "also"): bqr_geqrf_batched + bqr_apply_qh_batched on
     256 240x66 complex64 STAP matrices with one right-hand side each;
  C2 (under "also"): 1,000,000 4x4 fp32.
Inputs are seeded synthetic (bqr_inputs) and resident in HBM; before every
timed step the working buffer is restored from a pristine copy and L2 is
flushed by writing a 2x-L2 buffer (both untimed); each step is bracketed by
CUDA events on the launching stream.  Multi-GPU: one process per GPU under
torchrun (`--gpus N` without a torchrun environment re-launches itself under
torch.distributed.run; a WORLD_SIZE that disagrees with --gpus is an error),
each rank factors its own seeded slice, no data-path collective; NCCL only
for barriers and the MAX of per-rank times.  The line's headline is weak
scaling (per-GPU batch fixed) and it also carries strong scaling (the
config's batch split over the ranks), the per-matrix latency floor (batch 1,
one per SM, one resident round) and the C5 size-sweep cells.

--impl reference times the fp64 CPU oracle (oracle/, the parity reference)
on the host cores on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import bqr_dist  # noqa: E402
import bqr_inputs  # noqa: E402
import bqr_metrics as bm  # noqa: E402

METRIC = "batched QR GFLOP/s & % roofline (5000×56×56 fp32; STAP 240×66 c64) @1/2/4/8 B200"
UNIT = "GFLOP/s"
PROFILE_TRAFFIC = os.path.join(ROOT, "profiles", "traffic.json")


# --------------------------------------------------------------------- utils

env_rank = bqr_dist.env_rank


class ClockSampler:
    """NVML sampling of SM clock + throttle reasons during the timed region
    (the B200_PROFILING.md clocks line)."""

    REASONS = {
        0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
        0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
        0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting",
    }

    def __init__(self, device_index: int, period_s: float = 0.01):
        self.dev = device_index
        self.period = period_s
        self.samples = []
        self.reasons = 0
        self.max_mhz = None
        self._stop = threading.Event()
        self._t = None
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover - no NVML
            self.err = str(e)

    def _run(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                self.reasons |= nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.ok:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self):
        if not self.ok:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvml_unavailable"]}
        names = [n for b, n in self.REASONS.items() if self.reasons & b and n != "gpu_idle"]
        med = float(np.median(self.samples)) if self.samples else None
        return {"sm_mhz": med, "sm_max_mhz": self.max_mhz, "reasons": names, "samples": len(self.samples)}


def load_traffic(name: str, kernel: str | None = None):
    """DRAM bytes per launch of config `name` from the committed ncu capture;
    None when the capture was taken of another kernel class than the one the
    dispatch picks now."""
    try:
        with open(PROFILE_TRAFFIC) as f:
            t = json.load(f)
    except OSError:
        return None
    cls = t.get("_detail", {}).get(name, {}).get("class")
    if kernel is not None and cls is not None and cls != kernel:
        return None
    return t.get(name)


# --------------------------------------------------------------------- GPU arm

class Workload:
    """Device buffers for one config on one rank."""

    def __init__(self, name, rank, world, torch, bqr, batch=None, cfg=None, scaling="weak"):
        cfg = dict(bqr_inputs.CONFIGS[name] if cfg is None else cfg)
        self.name = name
        self.m, self.n, self.dt = cfg["m"], cfg["n"], cfg["dtype"]
        total = cfg["batch"] if batch is None else batch
        self.k = min(self.m, self.n)
        self.nrhs = cfg.get("nrhs", 0)
        self.torch, self.bqr = torch, bqr
        self.kind = cfg.get("kind", "qr")
        if scaling == "weak":
            # rank r owns matrices [r*B, (r+1)*B) of a world*B seeded stream
            lo, hi = bqr_dist.rank_slice(rank, world, total)
            stream_len = world * total
        else:
            # strong: the B matrices of the config split floor(r B / P) .. floor((r+1) B / P)
            lo, hi = bqr_dist.rank_slice(rank, world, 0, weak=False, total=total)
            stream_len = total
        self.batch = hi - lo
        self.global_batch = world * total if scaling == "weak" else total
        if cfg is not None and name not in bqr_inputs.CONFIGS:
            host = bqr_inputs.random_batch(self.m, self.n, stream_len, self.dt, cfg["seed"], cfg["dist"],
                                           start=lo, stop=hi)
        else:
            host = bqr_inputs.config_batch(name, start=lo, stop=hi, batch=stream_len)
        self.host = host
        self.pristine = torch.from_numpy(host).cuda()
        self.A = torch.empty_like(self.pristine)
        tdt = self.pristine.dtype
        self.tau = torch.empty((self.batch, self.k), dtype=tdt, device="cuda")
        if self.nrhs:
            Bh = bqr_inputs.rhs_batch(self.m, self.nrhs, stream_len, self.dt, cfg["seed"], start=lo, stop=hi)
            self.Bp = torch.from_numpy(Bh).cuda()
            self.B = torch.empty_like(self.Bp)
        self.code = bqr.R32 if self.dt == "f32" else bqr.C64
        self.stream = torch.cuda.current_stream()
        self.sptr = self.stream.cuda_stream
        lib = bqr.load()
        self.lib = lib
        import ctypes
        self.c = ctypes
        self.flops = self.batch * bm.geqrf_flops(self.m, self.n, self.dt)
        self.bytes = self.batch * bm.geqrf_bytes(self.m, self.n, self.dt)
        if self.kind != "qr":  # NEXT-3: LU / Gauss-Jordan
            self.info = torch.empty((self.batch,), dtype=torch.int32, device="cuda")
            if self.kind == "lu":
                self.flops = self.batch * bm.lu_flops(self.m, self.n, self.dt)
                self.bytes = self.batch * bm.lu_bytes(self.m, self.n, self.dt)
            else:
                self.flops = self.batch * bm.gj_flops(self.n, self.dt)
                self.bytes = self.batch * bm.gj_bytes(self.n, self.nrhs, self.dt)
            self.flops_apply = self.bytes_apply = 0
        elif self.nrhs:
            self.flops_apply = self.batch * bm.apply_flops(self.m, self.n, self.nrhs, self.dt)
            self.bytes_apply = self.batch * bm.apply_bytes(self.m, self.nrhs, self.dt)
        else:
            self.flops_apply = self.bytes_apply = 0

    def step_flops_total(self):
        """Useful flops of one step over the WHOLE job (all ranks)."""
        per = (self.flops + self.flops_apply) / max(1, self.batch)
        return per * self.global_batch

    def restore(self):
        self.A.copy_(self.pristine)
        if self.nrhs:
            self.B.copy_(self.Bp)

    def geqrf(self):
        c = self.c
        if self.kind == "lu":
            st = self.lib.bqr_getrf_np_batched(self.code, self.m, self.n, self.batch, c.c_void_p(self.A.data_ptr()),
                                               self.m, c.c_void_p(self.info.data_ptr()), c.c_void_p(self.sptr))
            if st:
                raise RuntimeError(f"bqr_getrf_np_batched -> {st}")
            return
        if self.kind == "gj":
            st = self.lib.bqr_gauss_jordan_batched(self.code, self.n, self.nrhs, self.batch,
                                                   c.c_void_p(self.A.data_ptr()), self.n, c.c_void_p(self.B.data_ptr()),
                                                   self.n, c.c_void_p(self.info.data_ptr()), c.c_void_p(self.sptr))
            if st:
                raise RuntimeError(f"bqr_gauss_jordan_batched -> {st}")
            return
        st = self.lib.bqr_geqrf_batched(self.code, self.m, self.n, self.batch, c.c_void_p(self.A.data_ptr()),
                                        self.m, c.c_void_p(self.tau.data_ptr()), c.c_void_p(self.sptr))
        if st:
            raise RuntimeError(f"bqr_geqrf_batched -> {st}")

    def geqrf_qhb(self):
        """Fused factorisation + Q^H b (one kernel for the STAP shape)."""
        c = self.c
        st = self.lib.bqr_geqrf_qhb_batched(self.code, self.m, self.n, self.nrhs, self.batch,
                                            c.c_void_p(self.A.data_ptr()), self.m, c.c_void_p(self.tau.data_ptr()),
                                            c.c_void_p(self.B.data_ptr()), self.m, c.c_void_p(self.sptr))
        if st:
            raise RuntimeError(f"bqr_geqrf_qhb_batched -> {st}")

    def apply(self):
        c = self.c
        st = self.lib.bqr_apply_qh_batched(self.code, self.m, self.n, self.k, self.nrhs, self.batch,
                                           c.c_void_p(self.A.data_ptr()), self.m, c.c_void_p(self.tau.data_ptr()),
                                           c.c_void_p(self.B.data_ptr()), self.m, c.c_void_p(self.sptr))
        if st:
            raise RuntimeError(f"bqr_apply_qh_batched -> {st}")


def barrier(torch, dist, world):
    bqr_dist.barrier(torch, dist)


def max_over_ranks(torch, dist, world, x: float) -> float:
    return bqr_dist.max_over_ranks(torch, dist, x)


# context only (another machine): the paper's Table VII GPU GFLOP/s
PAPER_TABLE_VII = {"S80": 134.0, "S192": 98.0}


def time_workload(w: Workload, steps: int, warmup: int, torch, dist, world, flush, sampler=None, fused=True):
    """Returns (ms_per_step, ms_of_the_factorisation_kernel).  With right-hand
    sides the step is the fused factorisation + Q^H b (one kernel, the
    augmented [A | b] of P:L313) unless fused=False (geqrf, then apply)."""
    ev = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(steps)]

    def run_step(i=None):
        if i is not None:
            ev[i][0].record(w.stream)
        if w.nrhs and fused and w.kind == "qr":
            w.geqrf_qhb()
            if i is not None:
                ev[i][1].record(w.stream)
        else:
            w.geqrf()
            if i is not None:
                ev[i][1].record(w.stream)
            if w.nrhs and w.kind == "qr":
                w.apply()
        if i is not None:
            ev[i][2].record(w.stream)

    for _ in range(warmup):
        w.restore()
        flush.zero_()
        run_step()
    barrier(torch, dist, world)
    ctx = sampler if sampler is not None else _Null()
    with ctx:
        for i in range(steps):
            w.restore()
            flush.zero_()
            run_step(i)
        barrier(torch, dist, world)
    step_ms = sum(e[0].elapsed_time(e[2]) for e in ev) / steps
    qr_ms = sum(e[0].elapsed_time(e[1]) for e in ev) / steps
    return max_over_ranks(torch, dist, world, step_ms), max_over_ranks(torch, dist, world, qr_ms)


class _Null:
    def __enter__(self):
        return self

    def __exit__(self, *a):
        pass


def roofline_obj(w: Workload, qr_ms: float, peaks: dict, n_sm: int, fused: bool = False):
    """Roofline of the dominant kernel (the geqrf launch, or the fused
    geqrf + Q^H b launch for configs with right-hand sides): SURVEY 8(d)."""
    hbm = float(peaks["hbm_gbs"])
    fp32 = bm.fp32_peak_tflops(n_sm, float(peaks.get("sm_max_mhz", 1965.0)))
    flops = w.flops + (w.flops_apply if fused else 0)
    nbytes = w.bytes + (w.bytes_apply if fused else 0)
    t_roof, bound = bm.roofline_time_s(flops, nbytes, hbm, fp32)
    t = qr_ms / 1e3
    kname = (w.bqr.load().bqr_lu_kernel_name(w.code, w.m, w.n, w.nrhs, int(w.kind == "gj")).decode()
             if w.kind != "qr" else
             w.bqr.load().bqr_qhb_kernel_name(w.code, w.m, w.n, w.nrhs).decode() if fused
             else w.bqr.kernel_name(w.code, w.m, w.n))
    traffic = load_traffic(w.name, kname)
    if bound == "hbm":
        ach, peak, unit = nbytes / t / 1e9, hbm, "GB/s"
    else:
        ach, peak, unit = flops / t / 1e12, fp32, "TFLOP/s"
    return {"bound": bound, "achieved": round(ach, 3), "peak": peak, "unit": unit,
            "frac": round(ach / peak, 4), "traffic": traffic,
            "peak_source": ("MEASURED_PEAKS.json hbm_gbs" if bound == "hbm" else
                            f"derived: {n_sm} SMs x 128 FP32 lanes x 2 x {peaks.get('sm_max_mhz', 1965.0)} MHz"),
            "roofline_us": round(t_roof * 1e6, 3), "kernel_us": round(qr_ms * 1e3, 3),
            "algorithmic_bytes": nbytes, "useful_flops": flops,
            "kernel": kname}


def e2e_host(w: Workload, steps: int, warmup: int, torch, dist, world):
    """Same metric end to end through the public host-buffer entry point
    (bqr_geqrf_batched_host): H2D of the step's inputs from pinned memory,
    the factorisation and D2H of R/V + tau all inside the timed region."""
    bqr = w.bqr
    host_in = torch.from_numpy(w.host.copy())
    Ah = torch.empty_like(host_in).pin_memory()
    tauh = torch.empty((w.batch, w.k), dtype=w.tau.dtype).pin_memory()
    chunk = max(1, w.batch // 4)  # tools/e2e_ab.py: //4 1.78 ms, //8 1.81, //16 2.06 (B200)
    wsb = bqr.host_workspace_bytes(w.code, w.m, w.n, w.m, chunk)
    ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
    ev = [[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in range(steps)]
    for _ in range(warmup):
        Ah.copy_(host_in)
        bqr.geqrf_batched_host(w.code, w.m, w.n, w.batch, Ah.data_ptr(), w.m, tauh.data_ptr(), ws.data_ptr(), wsb)
    barrier(torch, dist, world)
    for i in range(steps):
        Ah.copy_(host_in)  # restore the host input (untimed)
        ev[i][0].record(w.stream)
        bqr.geqrf_batched_host(w.code, w.m, w.n, w.batch, Ah.data_ptr(), w.m, tauh.data_ptr(), ws.data_ptr(), wsb)
        ev[i][1].record(w.stream)
    barrier(torch, dist, world)
    ms = max_over_ranks(torch, dist, world, sum(e[0].elapsed_time(e[1]) for e in ev) / steps)
    h2d = w.A.numel() * w.A.element_size()
    d2h = h2d + w.tau.numel() * w.tau.element_size()
    return ms, h2d, d2h


def cpu_baseline(name: str, min_seconds: float = 2.0, max_matrices: int | None = None):
    """The fp64 oracle, as it stands, on a bounded sample: the median of 3
    timed trials on all host cores, plus one trial on 1 core."""
    import oracle
    cfg = bqr_inputs.CONFIGS[name]
    b = cfg["batch"] if max_matrices is None else min(cfg["batch"], max_matrices)
    A = bqr_inputs.random_batch(cfg["m"], cfg["n"], cfg["batch"], cfg["dtype"], cfg["seed"], cfg["dist"], stop=b)
    per = bm.geqrf_flops(cfg["m"], cfg["n"], cfg["dtype"])

    def trial(Ab, secs):
        reps, t0 = 0, time.perf_counter()
        while True:
            oracle.geqrf_cm(Ab, cfg["m"], with_margin=False)
            reps += 1
            el = time.perf_counter() - t0
            if el >= secs:
                return reps * Ab.shape[0] / el  # matrices / s

    oracle.set_threads(0)
    oracle.geqrf_cm(A, cfg["m"], with_margin=False)  # warm (page-in, threads)
    rates = sorted(trial(A, min_seconds / 2) for _ in range(3))
    cores = oracle.max_threads()
    oracle.set_threads(1)
    one = trial(A[: max(1, b // 16)], min_seconds / 4)
    oracle.set_threads(0)
    med = rates[1]
    return {"value": round(med * per / 1e9, 4), "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"{b} of the {name} matrices ({cfg['m']}x{cfg['n']} {cfg['dtype']}), median of 3 trials of "
                      f"~{min_seconds / 2:.1f} s on {cores} threads; 1-core trial on {max(1, b // 16)} matrices; "
                      f"fp64 C oracle (OpenMP)",
            "matrices_per_s": round(med, 1), "trials_gflops": [round(r * per / 1e9, 4) for r in rates],
            "value_1core": round(one * per / 1e9, 4)}


def config_block(w: Workload, world, l2_note):
    op = {"qr": "geqrf" + (f" + Q^H b ({w.nrhs} rhs)" if w.nrhs else ""),
          "lu": "LU without pivoting (diagonally dominant)",
          "gj": f"Gauss-Jordan [A | b] ({w.nrhs} rhs, diagonally dominant)"}[w.kind]
    return {"workload": f"{w.name}: {w.batch} x {w.m}x{w.n} {w.dt} {op} per GPU", "m": w.m, "n": w.n,
            "batch_per_gpu": w.batch, "global_batch": w.global_batch,
            "dtype": w.dt, "l2": l2_note, "parallelism": f"dp{world} (independent matrices per rank)",
            "kernel": (w.bqr.load().bqr_qhb_kernel_name(w.code, w.m, w.n, w.nrhs).decode() if w.nrhs and w.kind == "qr"
                       else w.bqr.kernel_name(w.code, w.m, w.n) if w.kind == "qr" else "lu_rf_kernel")}


def latency_scan(w: Workload, torch, dist, world, flush, n_sm: int) -> dict:
    """Per-matrix latency floor: kernel time of a batch of
    1 matrix, of one matrix per SM and of one full round of resident matrices
    (bqr_resident_matrices), L2 flushed, max over ranks."""
    res = int(w.lib.bqr_resident_matrices(w.code, w.m, w.n))
    out = {"resident_matrices": res}
    full = w.batch
    for label, b in (("batch_1", 1), ("batch_n_sm", n_sm), ("batch_resident", res)):
        if b <= 0 or b > full:
            continue
        w.batch = b
        _, q_ms = time_workload(w, 20, 3, torch, dist, world, flush)
        out[f"{label}_us"] = round(q_ms * 1e3, 2)
    w.batch = full
    return out


C5_CELLS = [(16, "f32"), (56, "f32"), (128, "f32"), (256, "f32"), (16, "c64"), (56, "c64"), (128, "c64"),
            (256, "c64")]


def colnorm_check(w: Workload, torch, stride: int = 97) -> dict:
    """Property check that holds at any size (Q is unitary): ||R e_j|| equals
    ||A e_j|| on every `stride`-th matrix plus the first and the last
    (plain torch on the bench's own output; the oracle parity of the C5 cells
    at these batch sizes is tests/test_gpu_c5.py)."""
    w.restore()
    w.geqrf()
    torch.cuda.synchronize()
    idx = sorted(set(range(0, w.batch, stride)) | {w.batch - 1})
    A = w.pristine[idx].to(torch.complex128 if w.dt == "c64" else torch.float64)  # (s, n, m) storage
    R = w.A[idx].to(A.dtype)
    # storage [b, col, row]: upper triangle of the logical matrix = row <= col
    rows = torch.arange(w.m, device=A.device)[None, None, :]
    cols = torch.arange(w.n, device=A.device)[None, :, None]
    Rt = torch.where(rows <= cols, R, torch.zeros_like(R))
    na = torch.linalg.vector_norm(A, dim=2)
    nr = torch.linalg.vector_norm(Rt, dim=2)
    err = float(((nr - na).abs() / na.clamp_min(1e-30)).max())
    return {"sampled": len(idx), "colnorm_rel_err_max": err, "ok": err < 1e-5}


def run_c5(rank, world, torch, dist, bqr, flush, peaks, n_sm, l2_note, steps, warmup):
    cells = {}
    launches = 0
    for n, dt in C5_CELLS:
        cfg = bqr_inputs.c5_config(n, dt, n_sm=n_sm)
        name = f"C5_{dt}_{n}"
        w = Workload(name, rank, world, torch, bqr, cfg=cfg)
        k2 = max(3, min(steps, 50))
        s_ms, q_ms = time_workload(w, k2, warmup, torch, dist, world, flush)
        launches += k2 * int(w.lib.bqr_geqrf_launches(w.code, w.m, w.n, w.batch))
        cell = {"value": round(w.step_flops_total() / (s_ms / 1e3) / 1e9, 3), "unit": UNIT,
                "ms_per_step": round(s_ms, 6), "steps": k2,
                "matrices_per_s": round(w.global_batch / (s_ms / 1e3), 1),
                "config": config_block(w, world, l2_note),
                "roofline": roofline_obj(w, q_ms, peaks, n_sm),
                "check": colnorm_check(w, torch)}
        cells[name] = cell
        del w
        torch.cuda.empty_cache()
    return cells, launches


def dry_run(args, rank, world, torch, dist):
    """--dry-run: the rank / launch / slicing plumbing of a multi-GPU run
    without a GPU (gloo): every rank derives its weak and strong slices of
    the config, they are gathered over the process group, rank 0 prints them
    (tests/test_dist_gloo.py drives `bench.py --gpus 2 --dry-run`)."""
    if world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        dist.init_process_group("gloo")
    cfg = bqr_inputs.CONFIGS[args.config]
    weak = bqr_dist.rank_slice(rank, world, cfg["batch"])
    strong = bqr_dist.rank_slice(rank, world, 0, weak=False, total=cfg["batch"])
    t = bqr_dist.max_over_ranks(torch, dist, float(rank))
    got = bqr_dist.gather_ints(torch, dist, [rank, *weak, *strong])
    bqr_dist.barrier(torch, dist)
    if rank == 0:
        print(json.dumps({"dry_run": True, "n_gpus": world, "config": args.config, "max_rank": t,
                          "weak_slices": [g[1:3] for g in got], "strong_slices": [g[3:5] for g in got]}),
              flush=True)
    if world > 1:
        dist.destroy_process_group()


def run_ours(args):
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_andersonsk12_b200 as bqr
    rank, world, local = env_rank()
    if world != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world} (launch N ranks with torchrun, "
                         f"or run `python bench.py --gpus N` and let it re-launch itself)")
    if args.dry_run:
        return dry_run(args, rank, world, torch, dist)
    torch.cuda.set_device(local)
    if world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    bqr.load()
    props = torch.cuda.get_device_properties(local)
    n_sm = props.multi_processor_count
    l2 = props.L2_cache_size
    flush = torch.empty(2 * max(l2, 64 << 20), dtype=torch.uint8, device="cuda")
    l2_note = f"L2 flushed before every timed step by writing {flush.numel() >> 20} MiB (2x L2); input restored from a pristine copy (untimed)"
    peaks = bm.load_peaks()

    main = Workload(args.config, rank, world, torch, bqr, scaling=args.scaling)
    sampler = ClockSampler(local, 0.002)
    step_ms, qr_ms = time_workload(main, args.steps, args.warmup, torch, dist, world, flush, sampler)
    value = main.step_flops_total() / (step_ms / 1e3) / 1e9
    out = {
        "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(step_ms, 6), "higher_is_better": True,
        "scaling": args.scaling,
        "vs_baseline": None, "dtype": "f32" if main.dt == "f32" else "c64", "data": "synthetic (seeded iid Gaussian, bqr_inputs)",
        "config": config_block(main, world, l2_note),
        "matrices_per_s": round(main.global_batch / (step_ms / 1e3), 1),
        "roofline": roofline_obj(main, qr_ms, peaks, n_sm, fused=bool(main.nrhs)),
        "gpu_launches": args.steps * int(main.lib.bqr_geqrf_launches(main.code, main.m, main.n, main.batch)),
        "clocks": sampler.summary(),
    }
    # the other scaling mode at this N (both curves per run)
    other = "strong" if args.scaling == "weak" else "weak"
    ow = Workload(args.config, rank, world, torch, bqr, scaling=other)
    o_ms, o_q = time_workload(ow, max(3, min(args.steps, 100)), args.warmup, torch, dist, world, flush)
    out[other] = {"value": round(ow.step_flops_total() / (o_ms / 1e3) / 1e9, 3), "unit": UNIT,
                  "ms_per_step": round(o_ms, 6), "global_batch": ow.global_batch, "batch_per_gpu_max": ow.batch,
                  "matrices_per_s": round(ow.global_batch / (o_ms / 1e3), 1), "kernel_us": round(o_q * 1e3, 3)}
    out["gpu_launches"] += max(3, min(args.steps, 100))
    # per-matrix latency floor (strong-scaling limit)
    out["latency"] = latency_scan(ow if other == "weak" else main, torch, dist, world, flush, n_sm)
    del ow
    # end to end through the public host-buffer API
    e_steps = max(3, min(args.steps, 20))
    e_ms, h2d, d2h = e2e_host(main, e_steps, 2, torch, dist, world)
    out["e2e"] = {"value": round(main.global_batch * (main.flops / max(1, main.batch)) / (e_ms / 1e3) / 1e9, 3),
                  "unit": UNIT, "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h, "steps": e_steps,
                  "api": "bqr_geqrf_batched_host (pinned host buffers, chunked H2D/compute/D2H overlap)",
                  "ms_per_step": round(e_ms, 4)}
    if not args.no_also:
        also = {}
        for name in [c for c in ("C4", "C2", "S80", "S192", "L56", "GJ56") if c != args.config]:
            w = Workload(name, rank, world, torch, bqr, scaling=args.scaling)
            k2 = max(3, min(args.steps, 100))
            s_ms, q_ms = time_workload(w, k2, max(3, args.warmup), torch, dist, world, flush)
            also[name] = {"value": round(w.step_flops_total() / (s_ms / 1e3) / 1e9, 3), "unit": UNIT,
                          "ms_per_step": round(s_ms, 6), "steps": k2,
                          "matrices_per_s": round(w.global_batch / (s_ms / 1e3), 1),
                          "config": config_block(w, world, l2_note),
                          "roofline": roofline_obj(w, q_ms, peaks, n_sm, fused=bool(w.nrhs) and w.kind == "qr")}
            if name in PAPER_TABLE_VII:
                also[name]["paper_quadro6000_gflops"] = PAPER_TABLE_VII[name]
            out["gpu_launches"] += k2
            if name == "C4":
                also[name]["latency"] = latency_scan(w, torch, dist, world, flush, n_sm)
            if w.nrhs and w.kind == "qr":
                # context: the same step as two launches (geqrf, then apply_qh)
                s2, q2 = time_workload(w, k2, max(3, args.warmup), torch, dist, world, flush, fused=False)
                also[name]["unfused_two_launch"] = {"ms_per_step": round(s2, 6), "geqrf_ms": round(q2, 6),
                                                    "apply_ms": round(s2 - q2, 6)}
                out["gpu_launches"] += 2 * k2
            del w
        out["also"] = also
        if not args.no_c5:
            cells, nl = run_c5(rank, world, torch, dist, bqr, flush, peaks, n_sm, l2_note, args.steps,
                               max(3, args.warmup))
            out["c5"] = cells
            out["gpu_launches"] += nl
    # determinism evidence (outside the timed region): checksum of one
    # factorised slice per rank, gathered over the process group
    main.restore()
    main.geqrf()
    torch.cuda.synchronize()
    sums = bqr_dist.gather_ints(torch, dist, [bqr_dist.checksum(main.A.cpu().numpy())])
    out["checksums"] = [s[0] for s in sums]
    if rank == 0 and world == 1 and not args.no_cpu:
        out["cpu_baseline"] = cpu_baseline(args.config)
    if rank == 0:
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def run_reference(args):
    """--impl reference: the fp64 CPU oracle on the host cores (rank 0 only)."""
    rank, world, _ = env_rank()
    if rank != 0:
        return
    import oracle
    cfg = bqr_inputs.CONFIGS[args.config]
    sample = max(1, min(cfg["batch"], int(os.environ.get("BQR_REF_SAMPLE", 500 if cfg["m"] >= 32 else 20000))))
    A = bqr_inputs.random_batch(cfg["m"], cfg["n"], cfg["batch"], cfg["dtype"], cfg["seed"], cfg["dist"], stop=sample)
    oracle.set_threads(0)
    for _ in range(args.warmup):
        oracle.geqrf_cm(A, cfg["m"], with_margin=False)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.geqrf_cm(A, cfg["m"], with_margin=False)
    el = time.perf_counter() - t0
    flops = sample * bm.geqrf_flops(cfg["m"], cfg["n"], cfg["dtype"])
    value = flops * args.steps / el / 1e9
    cores = oracle.max_threads()
    desc = f"{sample} of the {args.config} matrices per step ({cfg['m']}x{cfg['n']} {cfg['dtype']} widened to fp64)"
    out = {"metric": METRIC, "value": round(value, 4), "unit": UNIT, "impl": "reference", "n_gpus": world,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(el / args.steps * 1e3, 4),
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
           "data": "synthetic (seeded iid Gaussian, bqr_inputs)",
           "config": {"workload": f"{args.config}: {cfg['m']}x{cfg['n']} {cfg['dtype']} geqrf (bounded sample)",
                      "sample_matrices": sample},
           "cpu_baseline": {"value": round(value, 4), "unit": UNIT, "cores": cores, "kind": "oracle", "sample": desc},
           "e2e": {"value": round(value, 4), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


def relaunch_under_torchrun(args) -> int:
    """`python bench.py --gpus N` without a torchrun environment: start N
    ranks (one process per GPU) on this node through torch.distributed.run,
    with the same arguments; rank 0 prints the JSON line."""
    import socket
    import subprocess
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C3", choices=["C1", "C2", "C3", "C4", "S80", "S192", "L56", "GJ56"])
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"],
                    help="headline mode; the line also carries the other mode at the same N")
    ap.add_argument("--no-also", action="store_true")
    ap.add_argument("--no-c5", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--dry-run", action="store_true", help="rank/slicing plumbing only (no GPU, gloo)")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.gpus < 1:
        raise SystemExit("--gpus must be >= 1")
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(relaunch_under_torchrun(args))
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()

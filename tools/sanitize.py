"""Small invocations of every kernel family through the C ABI, for
compute-sanitizer (tier 5):

    compute-sanitizer --tool memcheck  --error-exitcode 9 python tools/sanitize.py
    compute-sanitizer --tool racecheck --error-exitcode 9 python tools/sanitize.py
    compute-sanitizer --tool synccheck --error-exitcode 9 python tools/sanitize.py
    compute-sanitizer --tool initcheck --error-exitcode 9 python tools/sanitize.py

Each case uses a batch just above the persistent grid where the kernel runs
a persistent loop (so the prefetch / tile-swap / buffer-rotation paths run
for more than one matrix per CTA or warp).  Statuses are checked; numerics
are the parity tests' job.  `--quick` runs a reduced case list (racecheck
is slow).
"""
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bqr_inputs  # noqa: E402
import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402

QUICK = "--quick" in sys.argv
lib = bqr.load()
torch.cuda.set_device(0)
S = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
P = ctypes.c_void_p


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def code(dt):
    return bqr.R32 if dt == "f32" else bqr.C64


def geqrf(dt, m, n, batch):
    A = dev(bqr_inputs.random_batch(m, n, batch, dt, seed=m * 7 + n))
    tau = torch.empty((batch, min(m, n)), dtype=A.dtype, device="cuda")
    st = lib.bqr_geqrf_batched(code(dt), m, n, batch, P(A.data_ptr()), m, P(tau.data_ptr()), S)
    assert st == 0, ("geqrf", dt, m, n, st)
    return A, tau


def case_geqrf(dt, m, n, batch):
    A, tau = geqrf(dt, m, n, batch)
    torch.cuda.synchronize()
    return f"geqrf {dt} {m}x{n} x{batch} [{bqr.kernel_name(code(dt), m, n)}]"


def case_orgqr_apply(dt, m, n, batch, nrhs=2):
    A, tau = geqrf(dt, m, n, batch)
    B = dev(bqr_inputs.rhs_batch(m, nrhs, batch, dt, seed=3))
    st = lib.bqr_apply_qh_batched(code(dt), m, n, min(m, n), nrhs, batch, P(A.data_ptr()), m, P(tau.data_ptr()),
                                  P(B.data_ptr()), m, S)
    assert st == 0, ("apply", st)
    st = lib.bqr_orgqr_batched(code(dt), m, n, min(m, n), batch, P(A.data_ptr()), m, P(tau.data_ptr()), S)
    assert st == 0, ("orgqr", st)
    torch.cuda.synchronize()
    return f"apply_qh + orgqr {dt} {m}x{n} x{batch}"


def case_qhb_gels(dt, m, n, batch, nrhs=1):
    A = dev(bqr_inputs.random_batch(m, n, batch, dt, seed=5))
    B = dev(bqr_inputs.rhs_batch(m, nrhs, batch, dt, seed=6))
    tau = torch.empty((batch, n), dtype=A.dtype, device="cuda")
    info = torch.empty((batch,), dtype=torch.int32, device="cuda")
    st = lib.bqr_gels_batched(code(dt), m, n, nrhs, batch, P(A.data_ptr()), m, P(tau.data_ptr()), P(B.data_ptr()), m,
                              P(info.data_ptr()), S)
    assert st == 0, ("gels", st)
    torch.cuda.synchronize()
    return f"gels (fused geqrf+Q^H b, back substitution) {dt} {m}x{n} x{batch}"


def case_lu_gj(dt, n, batch, nrhs=1):
    A = dev(bqr_inputs.diag_dominant_batch(n, batch, dt, seed=n))
    info = torch.empty((batch,), dtype=torch.int32, device="cuda")
    st = lib.bqr_getrf_np_batched(code(dt), n, n, batch, P(A.data_ptr()), n, P(info.data_ptr()), S)
    assert st == 0, ("getrf_np", st)
    A = dev(bqr_inputs.diag_dominant_batch(n, batch, dt, seed=n + 1))
    B = dev(bqr_inputs.rhs_batch(n, nrhs, batch, dt, seed=n + 2))
    st = lib.bqr_gauss_jordan_batched(code(dt), n, nrhs, batch, P(A.data_ptr()), n, P(B.data_ptr()), n,
                                      P(info.data_ptr()), S)
    assert st == 0, ("gauss_jordan", st)
    torch.cuda.synchronize()
    return f"getrf_np + gauss_jordan {dt} {n}x{n} x{batch}"


def case_host(dt, m, n, batch):
    A = torch.from_numpy(bqr_inputs.random_batch(m, n, batch, dt, seed=9)).pin_memory()
    tau = torch.empty((batch, min(m, n)), dtype=A.dtype).pin_memory()
    chunk = max(1, batch // 4)
    wsb = bqr.host_workspace_bytes(code(dt), m, n, m, chunk)
    ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
    bqr.geqrf_batched_host(code(dt), m, n, batch, A.data_ptr(), m, tau.data_ptr(), ws.data_ptr(), wsb)
    return f"geqrf_batched_host {dt} {m}x{n} x{batch}"


def case_wy(dt, m, n, batch):
    A = dev(bqr_inputs.random_batch(m, n, batch, dt, seed=11))
    tau = torch.empty((batch, min(m, n)), dtype=A.dtype, device="cuda")
    wsb = bqr.geqrf_wy_workspace_bytes(code(dt), m, n, m, batch)
    ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
    st = bqr.geqrf_wy_batched_ptr(code(dt), m, n, batch, A.data_ptr(), m, tau.data_ptr(), ws.data_ptr(), wsb)
    assert st == 0, ("wy", dt, m, n, st)
    torch.cuda.synchronize()
    return f"geqrf_wy {dt} {m}x{n} x{batch}"


CASES = [
    (case_geqrf, ("f32", 4, 4, 300)),          # tiny, thread per matrix
    (case_geqrf, ("c64", 8, 8, 100)),
    (case_geqrf, ("f32", 16, 16, 64)),         # sub-warp staged groups
    (case_geqrf, ("f32", 56, 56, 5100)),       # C3 left-looking class: > 17 pairs on some CTAs (warp loop)
    (case_geqrf, ("f32", 56, 56, 33)),         # odd batch: the spare half-warp repeats its neighbour
    (case_geqrf, ("f32", 33, 30, 40)),
    (case_geqrf, ("c64", 32, 32, 40)),         # warp groups
    (case_geqrf, ("f32", 80, 80, 20)),         # CTA groups, named barriers
    (case_geqrf, ("c64", 96, 96, 20)),
    (case_geqrf, ("c64", 240, 66, 150)),       # C4 class: decoupled mbarriers, lazy rest, > 1 matrix per CTA
    (case_geqrf, ("c64", 80, 16, 40)),         # STAP 80x16 warp class
    (case_geqrf, ("c64", 192, 96, 150)),       # STAP 192x96 (R = 32)
    (case_geqrf, ("f32", 256, 256, 4)),        # single-SM 256 class
    (case_geqrf, ("c64", 224, 224, 3)),        # compact WY (a6/a9): panels + tcgen05 GEMMs + xLARFT
    (case_geqrf, ("c64", 225, 225, 3)),        # odd rows: tiled panels (a9)
    (case_geqrf, ("c64", 112, 112, 20)),       # R16G16 7x7 CTA class (97..112)
    (case_wy, ("f32", 256, 256, 3)),           # compact WY, fp32, caller workspace
    (case_orgqr_apply, ("f32", 56, 56, 30)),
    (case_orgqr_apply, ("c64", 240, 66, 10)),
    (case_qhb_gels, ("c64", 240, 66, 150)),    # fused augmented class (persistent loop)
    (case_qhb_gels, ("f32", 100, 37, 20)),
    (case_lu_gj, ("f32", 56, 40)),             # LU / GJ warp class
    (case_lu_gj, ("c64", 56, 10)),             # CTA class
    (case_lu_gj, ("f32", 8, 70)),
    (case_host, ("f32", 56, 56, 300)),
]
if QUICK:
    CASES = [c for i, c in enumerate(CASES) if i in (0, 3, 4, 7, 9, 13, 14, 15, 19, 21, 24)]
if "--new" in sys.argv:
    # this session's kernels only: the left-looking C3 class, and (run with
    # BQR_FORCE_VARIANT=alt_llc_c64_240x66_left3[_aug]) the C4 experiment
    CASES = [(case_geqrf, ("f32", 56, 56, 5100)), (case_geqrf, ("f32", 56, 56, 33)),
             (case_geqrf, ("c64", 240, 66, 300)), (case_qhb_gels, ("c64", 240, 66, 300))]

for fn, args in CASES:
    print("ok", fn(*args), flush=True)
print("all cases launched and synchronised")

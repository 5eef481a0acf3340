"""bqr_model -- NEXT-4: the paper's per-column performance
model, and the same model re-parameterised for the B200 register-file
kernels.  Measurement/diagnostics only: no method arithmetic.

The paper (Sec. V-D, Table VI) costs one column of a
one-problem-per-block QR as

  Column   N g (norm) + (1 + sqrt p) b + sqrt p g (thread-0 reduction)
           + g_sqrt + 2 g_div + 2 g (scale factor) + 2 b (write/read it)
           + N g + N b + a_sync (scale the column, write it to shared)
  Trailing N b (read v) + N^2 g (matvec) + 2 a_sync + (1 + sqrt p) b
           + sqrt p g (matvec reduction) + N b + N^2 g + a_sync (rank-1)

with N the rows per thread of the live sub-matrix, g the FP pipeline
latency, b a shared-memory access, a_sync a block barrier (Table IV:
g = 18, shared latency 27, a_sync = 46 cycles on the Quadro 6000), summed
over the n - 1 columns; LU per column: g_div + a_sync + 2 b + N g
+ 2 N b + a_sync + 2 N b + N^2 g + a_sync.  ``paper_qr_cycles`` /
``paper_lu_cycles`` evaluate it (readings: b = the 27-cycle shared latency,
g_sqrt = g_div = 2 g: the paper took them from a GT200 study it does not
print); the paper measured 150,203 (QR) and 68,250 (LU) compute cycles for
56 x 56 (Table V).

On B200 the kernels replace the thread-0 serial reductions by shuffle
butterflies and overlap the reflector chain with the trailing update
(look-ahead), so the model has two parts per column k:

  chain_k  the dependent latency from v_k to v_{k+1}: shared-memory read,
           the slot-P dot (FMA chain), log2 R shuffle+add levels, the
           update, the norm (FMA chain + log2 R levels + the alpha
           shuffle), the IEEE sqrt/div chain, the publish (shared write +
           signal);
  issue_k  warp instructions a scheduler must issue for its resident
           groups: 2 Nr Nc FMA instructions per lane (FFMA2 halves them
           for complex), the reduction shuffles/adds, and a per-step
           overhead O (masks, loads, scalar chain) calibrated from ncu's
           executed-instruction count of the bench kernel.

A column then costs between max(chain_k, issue_k) (perfect overlap, IPC 1
per scheduler) and chain_k + issue_k (no overlap); the kernel takes
rounds x sum_k of that.  Latencies come from ``tools/micro`` on B200
(``profiles/micro_r01.jsonl``): FFMA 4.24, shuffle+add 30.2, shared load
29.0, sqrt.rn + div.rn chain 118 cycles.
"""
from __future__ import annotations

import math
from dataclasses import dataclass

# Table IV, Quadro 6000; readings for the values it does not print
FERMI = dict(g=18.0, b=27.0, a_sync=46.0, g_sqrt=36.0, g_div=36.0)

# tools/micro on B200 (profiles/micro_r01.jsonl)
B200 = dict(l_fma=4.24, l_shfl_add=30.17, l_lds=29.02, l_sqrtdiv=118.06, f_ghz=1.965, schedulers=4)


def _panels(n_cols: int, width: int):
    """(columns in panel, panel index) for a 2D-cyclic layout with `width`
    column groups: panel P holds columns P*width .. P*width+width-1."""
    P = 0
    k = 0
    while k < n_cols:
        cnt = min(width, n_cols - k)
        yield cnt, P
        k += cnt
        P += 1


def paper_qr_cycles(n: int, p: int = 64, prm: dict = FERMI) -> float:
    """Table VI QR estimate for an n x n matrix on p threads (sqrt p x sqrt p
    grid), compute only, summed over the n - 1 columns."""
    g, b, a = prm["g"], prm["b"], prm["a_sync"]
    sp = int(round(math.sqrt(p)))
    total = 0.0
    for cnt, P in _panels(n - 1, sp):
        N = math.ceil(n / sp) - P  # rows (and columns) per thread in panel P
        col = N * g + (1 + sp) * b + sp * g + prm["g_sqrt"] + 2 * prm["g_div"] + 2 * g + 2 * b + N * g + N * b + a
        trail = N * b + N * N * g + 2 * a + (1 + sp) * b + sp * g + N * b + N * N * g + a
        total += cnt * (col + trail)
    return total


def paper_lu_cycles(n: int, p: int = 64, prm: dict = FERMI) -> float:
    """Table VI LU estimate (n - 1 columns)."""
    g, b, a = prm["g"], prm["b"], prm["a_sync"]
    sp = int(round(math.sqrt(p)))
    total = 0.0
    for cnt, P in _panels(n - 1, sp):
        N = math.ceil(n / sp) - P
        col = prm["g_div"] + a + 2 * b + N * g + 2 * N * b + a
        trail = 2 * N * b + N * N * g + a
        total += cnt * (col + trail)
    return total


@dataclass
class Layout:
    """A register-file class: R row lanes x G column groups per matrix,
    MR x NC elements per lane, `groups_per_warp` matrices per warp (sub-warp
    groups) or `warps` warps per matrix (CTA groups), `resident` matrices
    per SM, complex or real, overhead O instructions per lane-step."""
    m: int
    n: int
    R: int
    G: int
    MR: int
    NC: int
    cplx: bool
    resident: int           # matrices resident per SM
    warps_per_matrix: float  # 0.5 = two matrices per warp
    overhead: float         # per-step instructions besides FMAs and reductions
    packed: bool = False    # FFMA2 in the matvec / rank-1
    signal: float = 0.0     # extra cross-warp signal latency per column


def column_costs(L: Layout, lat: dict = B200):
    """Per-column (chain, issue-per-scheduler) cycle estimates."""
    r = int(round(math.log2(L.R))) if L.R > 1 else 0
    words = 2 if L.cplx else 1
    out = []
    kmax = min(L.m, L.n)
    for k in range(kmax):
        P = k // L.G
        i0 = (P * L.G) // L.R
        Nr = L.MR - i0
        Nc = L.NC - P
        fma_per_mac = (2 if L.packed else 4) if L.cplx else 1
        chain = (lat["l_lds"] + math.ceil(Nr / 4) * lat["l_fma"] * fma_per_mac + r * lat["l_shfl_add"] * words
                 + lat["l_fma"] + math.ceil(Nr / 4) * lat["l_fma"] + r * lat["l_shfl_add"] + lat["l_shfl_add"]
                 + lat["l_sqrtdiv"] * (1.5 if L.cplx else 1.0) + lat["l_lds"] + L.signal)
        per_lane = 2 * Nr * Nc * fma_per_mac + 2 * r * Nc * words + L.overhead
        warps_per_sched = L.resident * L.warps_per_matrix / lat["schedulers"]
        issue = per_lane * warps_per_sched
        out.append((chain, issue))
    return out


def predict_us(L: Layout, batch: int, n_sm: int = 148, lat: dict = B200) -> dict:
    """Kernel time bounds (us): rounds x sum over columns of max (overlap)
    and of the sum (no overlap); the last partial round is costed with the
    issue of its busiest SM (chain-bound when that is small)."""
    per_round = batch / (L.resident * n_sm)
    full = math.floor(per_round)
    frac = per_round - full
    cols = column_costs(L, lat)
    lo_full = sum(max(c, i) for c, i in cols)
    hi_full = sum(c + i for c, i in cols)
    # the last round: the busiest SM holds ceil(frac x resident) matrices
    share = math.ceil(frac * L.resident - 1e-9) / L.resident if frac > 0 else 0.0
    lo_part = sum(max(c, i * share) for c, i in cols) if frac > 0 else 0.0
    hi_part = sum(c + i * share for c, i in cols) if frac > 0 else 0.0
    f = lat["f_ghz"] * 1e3  # cycles per us
    return {"rounds": per_round, "lo_us": (full * lo_full + lo_part) / f, "hi_us": (full * hi_full + hi_part) / f,
            "chain_cycles": sum(c for c, _ in cols), "issue_cycles": sum(i for _, i in cols)}


# The bench kernels; overhead O calibrated from ncu's
# executed instructions of the same kernel (profiles/r01/details_*.txt).
C3_LAYOUT = Layout(m=56, n=56, R=4, G=4, MR=14, NC=14, cplx=False, resident=16, warps_per_matrix=0.5,
                   overhead=110.0)
C4_LAYOUT = Layout(m=240, n=66, R=32, G=11, MR=8, NC=6, cplx=True, resident=1, warps_per_matrix=11,
                   overhead=90.0, packed=True, signal=60.0)
# round 2: the left-looking C3 class (csrc/bqr_ll.cuh) -- the same 4 x 4
# lanes per matrix and per-column reflector chain, but only a <= 4-slot
# column block per lane and 34 matrices resident per SM (one round)
C3_LL_LAYOUT = Layout(m=56, n=56, R=4, G=4, MR=14, NC=4, cplx=False, resident=34, warps_per_matrix=0.5,
                      overhead=110.0, packed=True)
LAYOUTS = {"C3": C3_LAYOUT, "C3_LL": C3_LL_LAYOUT, "C4": C4_LAYOUT}


# ----------------------------------------------------------------------------
# Round 2: bounds that price the issue stalls (NEXT-4).
#
# Microbenchmarks on B200 (tools/micro/micro2.cu -> profiles/r02/micro2.jsonl,
# in-kernel clock64 cycles): FFMA latency 4.43, shuffle + add 30.3, shared
# load 29.0, IEEE sqrt + div chain 118, mbarrier hand-off between two warps
# 98, named barrier (64 threads) 29, __syncthreads 16 (32 thr) .. 77 (1024),
# cluster barrier 355-379, DSMEM remote load 202-226; FP32 pipe at 8-16
# resident warps: FFMA 92, FFMA2 83-88 FMA / clk / SM (of 128); shared
# memory 127.5 B / clk / SM (Table II analogue); an empty kernel between two
# CUDA events 4.96 us (min), 6.9 us (mean).
B200_R2 = dict(l_fma=4.43, l_shfl_add=30.33, l_lds=29.02, l_sqrtdiv=122.0, l_mbar=98.0, f_ghz=1.965,
               schedulers=4, fma_per_clk_sm=92.0, launch_event_us=4.96)


def bounds_us(L: Layout, batch: int, instr_total: float, cpi_warp: float, useful_fmas: float,
              n_sm: int = 148, lat: dict = B200_R2) -> dict:
    """Lower / upper bounds of one launch from measured counts.

    lo = the largest of three lower bounds: issue (every warp instruction of
         the launch, ncu ``inst_executed``, at 1 per scheduler per cycle),
         FP32 pipe (useful FMAs at the measured FFMA rate) and the reflector
         chain (rounds x sum of the per-column dependent latency, which no
         schedule can shorten);
    hi = ceil(rounds) x (the chain fully exposed + the instructions of one
         warp per round x the measured warp CPI, ncu "warp cycles per issued
         instruction", i.e. the issue stalls of this kernel at its
         occupancy, x the busiest scheduler's share of the SM's warps over
         the mean share): every round paid at full contention, the last
         (partial) one included, nothing of the chain hidden.
    The per-matrix latency floor (batch 1, the strong-scaling limit) is the
    chain plus one warp's instructions at CPI 1 (lo1) ... at the measured
    CPI (hi1).  The hi bounds add the measured launch / event overhead of an
    event-timed kernel (B200_R2["launch_event_us"])."""
    f = lat["f_ghz"] * 1e3
    slots = L.resident * n_sm
    rounds = batch / slots
    warps = max(1.0, batch * L.warps_per_matrix)             # warp-iterations of the launch
    per_warp_round = instr_total / warps                     # instructions of one warp per matrix group
    cols = column_costs(L, {**B200, **{k: v for k, v in lat.items() if k in B200}})
    chain = sum(c for c, _ in cols)
    issue = instr_total / (lat["schedulers"] * n_sm)
    fma = useful_fmas / (lat["fma_per_clk_sm"] * n_sm)
    lo = max(issue, fma, math.ceil(rounds - 1e-9) * chain)
    # the measured CPI is the mean over all warps; a scheduler holding
    # ceil(w/4) of an SM's w warps (17 warps: 5 on one, 4.25 on average)
    # stretches its warps' stalls by that ratio, and the launch lasts as long
    # as its slowest warp (profiles/r02/ll/timeline_full_batch.txt: the
    # 5-warp scheduler's warps finish ~10% after the others)
    wps = max(1.0, min(float(L.resident), batch / n_sm) * L.warps_per_matrix)
    per_sched = wps / lat["schedulers"]
    skew = max(1.0, math.ceil(per_sched - 1e-9) / per_sched) if per_sched >= 1.0 else 1.0
    hi = math.ceil(rounds - 1e-9) * (chain + per_warp_round * cpi_warp * skew)
    # an event-timed launch also carries the launch / event overhead (an
    # empty kernel measures 4.96 us min between two CUDA events on B200)
    return {"rounds": rounds, "lo_us": lo / f, "hi_us": hi / f + lat["launch_event_us"],
            "lo_terms_us": {"issue": issue / f, "fp32_pipe": fma / f, "chain": math.ceil(rounds - 1e-9) * chain / f},
            "chain_cycles_per_matrix": chain, "instr_per_warp_round": per_warp_round, "cpi_warp": cpi_warp,
            "scheduler_skew": skew,
            "latency_floor_us": {"lo": (chain + per_warp_round) / f,
                                 "hi": (chain + per_warp_round * cpi_warp) / f + lat["launch_event_us"]}}


S80_LAYOUT = Layout(m=80, n=16, R=16, G=4, MR=5, NC=4, cplx=True, resident=8, warps_per_matrix=2,
                    overhead=60.0, packed=True, signal=29.0)

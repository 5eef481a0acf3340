// bqr_launch.cuh -- host-side launch plumbing shared by the translation
// units of libbqr.so (split so the size-class instantiations compile in
// parallel): the per-call descriptor, the plan table entry, and the
// launch templates of the register-file, tiny and Q^H B kernels.
#pragma once
#include <cstdlib>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>

#include "../../include/bqr.h"
#include "bqr_apply.cuh"
#include "bqr_rf.cuh"
#include "bqr_tiny.cuh"

namespace bqr {
namespace host {

constexpr int kMaxDevices = 64;

inline int current_device() {
  int d = 0;
  cudaGetDevice(&d);
  return d < 0 ? 0 : (d >= kMaxDevices ? kMaxDevices - 1 : d);
}

// Raise a kernel's dynamic-smem limit once per (kernel, device) (bqr_api.cu).
bool ensure_smem(const void *kern, size_t smem);

inline int finish_launch() {
  return cudaGetLastError() == cudaSuccess ? BQR_SUCCESS : BQR_ERR_CUDA;
}

// ------------------------------------------------------------------ plans
struct Call {
  void *A;
  void *tau;
  long long batch;
  int m, n, k, lda;
  cudaStream_t stream;
  void *B = nullptr;  // fused Q^H B (augmented columns); direct-load classes only
  int ldb = 1, nrhs = 0;
  long long strideA = -1, strideT = -1;  // batch strides; -1 = LAPACK-contiguous
  // non-null: report how many matrices of this shape are resident on the
  // current device at once (occupancy x matrices per CTA) and launch nothing
  long long *resident = nullptr;
};

// occupancy-based residency of a kernel: CTAs per SM x SMs x matrices per CTA
inline long long resident_of(const void *kern, int threads, size_t smem, long long per_cta) {
  int sms = 0, bps = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, current_device());
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, kern, threads, smem);
  return (long long)sms * bps * per_cta;
}

using LaunchFn = int (*)(const Call &);

struct Plan {
  const char *name;
  LaunchFn geqrf;
  LaunchFn orgqr;
};

inline int staging_ld(int m) {
  // multiple of 4 floats so rows are 16-byte chunks
  return (m + 3) & ~3;
}

template <class T, int R, int G, int MR, int NC, int GPB, bool STAGE, bool EX, bool AUG, bool ORG, int MB = 1>
int launch_rf(const Call &c) {
  using Cfg = RfCfg<T, R, G, MR, NC, GPB, STAGE, EX>;
  if (EX && (c.m != R * MR || c.n != G * NC)) return BQR_ERR_NOT_SUPPORTED;
  if (c.nrhs > 0 && (!AUG || STAGE || EX || ORG || c.n + c.nrhs > G * NC)) return BQR_ERR_NOT_SUPPORTED;
  RfArgs a;
  a.A = c.A;
  a.tau = c.tau;
  a.batch = c.batch;
  a.lda = c.lda;
  a.m = c.m;
  a.n = c.n;
  a.kmax = c.k;
  a.ldS = STAGE ? staging_ld(c.m) : 0;
  a.tileWords = STAGE ? ((a.ldS * c.n + 3) & ~3) : 0;
  const bool aligned = (reinterpret_cast<uintptr_t>(c.A) & 15) == 0;
  a.vec4 = (STAGE && (c.lda % 4 == 0) && (c.m % 4 == 0) && aligned) ? 1 : 0;
  a.bulk = (STAGE && c.lda == c.m && a.ldS == c.m && aligned && ((size_t)c.m * c.n * sizeof(T)) % 16 == 0) ? 1 : 0;
  a.B = c.B;
  a.ldb = c.ldb;
  a.nrhs = c.nrhs;
  a.strideA = c.strideA >= 0 ? c.strideA : (long long)c.lda * c.n;
  a.strideT = c.strideT >= 0 ? c.strideT : (long long)c.k;
  a.strideB = (long long)c.ldb * c.nrhs;
  if (c.strideA >= 0) a.bulk = 0;  // panel views are not contiguous matrices
  // multi-warp geqrf kernels run a persistent matrix loop with a TMA-bulk
  // prefetch of the next contiguous matrix into a shared-memory tile
  constexpr bool kLoop = (R * G > 32) && !STAGE && !ORG;
  const size_t mat_bytes = (size_t)c.m * c.n * sizeof(T);
  const bool prefetch = kLoop && c.strideA == -1 && c.lda == c.m && aligned && mat_bytes % 16 == 0 &&
                        (size_t)Cfg::kSmallAll * 4 + mat_bytes <= 200 * 1024;
  if (kLoop) a.bulk = prefetch ? 1 : 0;
  const size_t smem = (size_t)Cfg::kSmallAll * 4 + (STAGE ? (size_t)GPB * a.tileWords * 4 : 0) +
                      (prefetch ? mat_bytes : 0);
  auto kern = ORG ? orgqr_rf_kernel<T, R, G, MR, NC, GPB, STAGE, EX, AUG, MB> : geqrf_rf_kernel<T, R, G, MR, NC, GPB, STAGE, EX, AUG, MB>;
  if (!ensure_smem(reinterpret_cast<const void *>(kern), smem)) return BQR_ERR_CUDA;
  if (c.resident) {
    *c.resident = resident_of(reinterpret_cast<const void *>(kern), Cfg::NT, smem, GPB);
    return BQR_SUCCESS;
  }
  long long grid = (c.batch + GPB - 1) / GPB;
  // sub-warp exact-shape kernels run a persistent prefetching warp loop when
  // the batch is contiguous (a.bulk)
  const bool warp_loop = (R * G <= 32) && (R * G * GPB == 32) && STAGE && EX && !ORG && a.bulk;
  if (prefetch || warp_loop) {
    // persistent grid: resident CTAs only (occupancy depends on smem, i.e.
    // on the shape, so it is queried per call; host-only, no sync)
    int sms = 0, bps = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, current_device());
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, kern, Cfg::NT, smem);
    static const int cap = [] {  // experiment knob: resident CTAs per SM
      const char *e = std::getenv("BQR_MAX_BPS");
      return e ? std::atoi(e) : 0;
    }();
    if (cap > 0) bps = std::min(bps, cap);
    grid = std::min<long long>(grid, std::max(1, sms * std::max(1, bps)));
  }
  if (grid > 0x7fffffffLL) return BQR_ERR_NOT_SUPPORTED;
  kern<<<(unsigned)grid, Cfg::NT, smem, c.stream>>>(a);
  return finish_launch();
}

template <class T, int M, int N>
int launch_tiny(const Call &c) {
  using K = Tiny<T, M, N>;
  TinyArgs a;
  a.A = c.A;
  a.tau = c.tau;
  a.batch = c.batch;
  a.lda = c.lda;
  a.staged = (K::kCanStage && c.lda == M && (reinterpret_cast<uintptr_t>(c.A) & 15) == 0) ? 1 : 0;
  const long long per_block = 32LL * K::kWarps;
  if (c.resident) {
    *c.resident = resident_of(reinterpret_cast<const void *>(geqrf_tiny_kernel<T, M, N>), K::kWarps * 32, 0, per_block);
    return BQR_SUCCESS;
  }
  const long long grid = (c.batch + per_block - 1) / per_block;
  if (grid > 0x7fffffffLL) return BQR_ERR_NOT_SUPPORTED;
  geqrf_tiny_kernel<T, M, N><<<(unsigned)grid, K::kWarps * 32, 0, c.stream>>>(a);
  return finish_launch();
}

// ---- size classes: smallest class that holds (m, n)
#define RF_PLAN_XA(T, R, G, MR, NC, GPB, STAGE, EX, AUG, NAME)             \
  Plan {                                                                 \
    NAME, &launch_rf<T, R, G, MR, NC, GPB, STAGE, EX, AUG, false>,       \
        &launch_rf<T, R, G, MR, NC, GPB, STAGE, EX, false, true>         \
  }
// MB > 1: register cap for MB resident CTAs per SM (launch bounds)
#define RF_PLAN_XM(T, R, G, MR, NC, GPB, STAGE, EX, MB, NAME)                  \
  Plan {                                                                     \
    NAME, &launch_rf<T, R, G, MR, NC, GPB, STAGE, EX, false, false, MB>,     \
        &launch_rf<T, R, G, MR, NC, GPB, STAGE, EX, false, true, MB>         \
  }
#define RF_PLAN_X(T, R, G, MR, NC, GPB, STAGE, EX, NAME) RF_PLAN_XA(T, R, G, MR, NC, GPB, STAGE, EX, false, NAME)
#define RF_PLAN(T, R, G, MR, NC, GPB, STAGE, NAME) RF_PLAN_X(T, R, G, MR, NC, GPB, STAGE, false, NAME)
// augmented (fused Q^H B) variant of a direct-load class
#define RF_PLAN_AUG(T, R, G, MR, NC, NAME) RF_PLAN_XA(T, R, G, MR, NC, 1, false, false, true, NAME)

struct ClassEntry {
  bqr_dtype_t dt;
  int mmax, nmax;           // class bounds (m <= mmax, n <= nmax)
  int exact_m, exact_n;     // > 0: preferred for exactly this shape
  bool alt;                 // alternative variant: only via BQR_FORCE_VARIANT
  Plan plan;
};

// Size classes.  Order matters: exact shapes first,
// then the smallest class that holds (m, n).
template <class T, int MR, int NB>
int launch_apply(const ApplyArgs &a, cudaStream_t s) {
  constexpr int PF = MR <= 2 ? 8 : 6;  // reflector columns in flight per warp
  using K = ApplyQh<T, MR, NB, PF>;
  const long long nblk = (a.nrhs + NB - 1) / NB;
  const long long items = a.batch * nblk;
  const long long grid = (items + K::kWarps - 1) / K::kWarps;
  if (grid > 0x7fffffffLL) return BQR_ERR_NOT_SUPPORTED;
  apply_qh_kernel<T, MR, NB, PF><<<(unsigned)grid, K::kWarps * 32, 0, s>>>(a);
  return finish_launch();
}

template <class T>
int apply_dispatch(const ApplyArgs &a, cudaStream_t s) {
  const int mr = (a.m + 31) / 32;
  if (mr <= 1) return launch_apply<T, 1, 4>(a, s);
  if (mr <= 2) return launch_apply<T, 2, 4>(a, s);
  if (mr <= 4) return launch_apply<T, 4, 2>(a, s);
  if (mr <= 8) return launch_apply<T, 8, 1>(a, s);
  return BQR_ERR_NOT_SUPPORTED;
}

// class tables (one translation unit each) and the tiny / apply entry points
const ClassEntry *classes_ll(int *n);
const ClassEntry *classes_llc(int *n);
const ClassEntry *classes_cl(int *n);
const ClassEntry *classes_co(int *n);
const ClassEntry *classes_headline(int *n);
const ClassEntry *classes_f32(int *n);
const ClassEntry *classes_c64(int *n);
const ClassEntry *classes_alt(int *n);
Plan tiny_plan_f32(int m, int n);
Plan tiny_plan_c64(int m, int n);
int apply_dispatch_f32(const ApplyArgs &a, cudaStream_t s);
int apply_dispatch_c64(const ApplyArgs &a, cudaStream_t s);
int launch_selftest_math(long long n, unsigned seed, unsigned long long *counts, cudaStream_t s);
// compact-WY blocked QR with tensor-core trailing updates (bqr_wy.cu)
int wy_panel_width(bqr_dtype_t dt);
bool wy_supported(bqr_dtype_t dt, int m, int n, int lda);
size_t wy_workspace_bytes(bqr_dtype_t dt, int m, int n, int chunk);
int geqrf_wy(bqr_dtype_t dt, int m, int n, long long batch, void *A, int lda, void *tau, void *work, size_t work_bytes,
             cudaStream_t stream, const Plan *(*pick_panel)(int, int));
size_t orgqr_wy_workspace_bytes(bqr_dtype_t dt, int m, int n, int k, int chunk);
int orgqr_wy(bqr_dtype_t dt, int m, int n, int k, long long batch, void *A, int lda, const void *tau, void *work,
             size_t work_bytes, cudaStream_t stream);
// back substitution X = R^{-1} C of the least-squares path (bqr_solve.cu)
int solve_upper_dispatch(bqr_dtype_t dt, const void *A, int lda, long long strideA, void *B, int ldb,
                         long long strideB, int *info, long long batch, int n, int nrhs, cudaStream_t s);

}  // namespace host
}  // namespace bqr

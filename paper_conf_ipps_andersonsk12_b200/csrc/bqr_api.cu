// bqr_api.cu -- host side of libbqr.so: the C ABI declared in include/bqr.h.
//
// Argument validation (LAPACK xerbla-style -i codes), quick returns, the
// size-class dispatch table (dtype, m, n) -> hand-written sm_100a kernel, one
// launch per call on the caller's stream, and the host-buffer streaming entry
// point.  No allocation per call, no host synchronisation (except the
// explicitly synchronous *_host entry), no state beyond per-device kernel
// attributes.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>

#include "../../include/bqr.h"
#include "bqr_apply.cuh"
#include "bqr_rf.cuh"
#include "bqr_tiny.cuh"

namespace {

using namespace bqr;

constexpr int kMaxDevices = 64;

int current_device() {
  int d = 0;
  cudaGetDevice(&d);
  return d < 0 ? 0 : (d >= kMaxDevices ? kMaxDevices - 1 : d);
}

// Raise a kernel's dynamic-smem limit once per (kernel, device).  Keyed by
// the kernel's address: every rf instantiation has the same function type.
bool ensure_smem(const void *kern, size_t smem) {
  if (smem <= 48 * 1024) return true;
  struct Entry {
    const void *k;
    int dev;
    size_t bytes;
  };
  static std::mutex mu;
  static Entry table[512];
  static int used = 0;
  const int d = current_device();
  std::lock_guard<std::mutex> lock(mu);
  for (int i = 0; i < used; ++i)
    if (table[i].k == kern && table[i].dev == d) {
      if (table[i].bytes >= smem) return true;
      if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
        return false;
      table[i].bytes = smem;
      return true;
    }
  if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
    return false;
  if (used < 512) table[used++] = Entry{kern, d, smem};
  return true;
}

int finish_launch() {
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
};

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

template <class T, int R, int G, int MR, int NC, int GPB, bool STAGE, bool EX, bool AUG, bool ORG>
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
  auto kern = ORG ? orgqr_rf_kernel<T, R, G, MR, NC, GPB, STAGE, EX, AUG> : geqrf_rf_kernel<T, R, G, MR, NC, GPB, STAGE, EX, AUG>;
  if (!ensure_smem(reinterpret_cast<const void *>(kern), smem)) return BQR_ERR_CUDA;
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
const ClassEntry kClasses[] = {
    // headline shapes, exact fits
    {BQR_R32, 56, 56, 56, 56, false, RF_PLAN_X(float, 4, 4, 14, 14, 2, true, true, "rf_f32_R4G4_14x14_x2_exact")},
    {BQR_C64, 240, 66, 240, 66, false, RF_PLAN(float2, 32, 11, 8, 6, 1, false, "rf_c64_R32G11_8x6_cta")},
    // augmented classes (fused Q^H B): 240x66 + up to 6 rhs, <=128 squares
    {BQR_C64, 256, 72, 240, 67, true, RF_PLAN_AUG(float2, 32, 12, 8, 6, "rf_c64_R32G12_8x6_aug")},
    {BQR_C64, 128, 128, 0, 0, true, RF_PLAN_AUG(float2, 32, 16, 4, 8, "rf_c64_R32G16_4x8_aug")},
    {BQR_R32, 128, 128, 0, 0, true, RF_PLAN_AUG(float, 32, 8, 4, 16, "rf_f32_R32G8_4x16_aug")},
    // alternatives kept for measurement (BQR_FORCE_VARIANT)
    {BQR_R32, 56, 56, 56, 56, true, RF_PLAN_X(float, 2, 8, 28, 7, 2, true, true, "rf_f32_R2G8_28x7_x2_exact")},
    {BQR_C64, 240, 66, 240, 66, true, RF_PLAN(float2, 32, 16, 8, 5, 1, false, "rf_c64_R32G16_8x5_cta")},
    // fp32 classes: square R x G lane grids where the register budget allows
    // (one pivot-mask row per panel), several matrices per warp when small
    {BQR_R32, 16, 16, 0, 0, false, RF_PLAN(float, 2, 2, 8, 8, 8, true, "rf_f32_R2G2_8x8_x8_stage")},
    {BQR_R32, 24, 24, 0, 0, false, RF_PLAN(float, 2, 2, 12, 12, 8, true, "rf_f32_R2G2_12x12_x8_stage")},
    {BQR_R32, 32, 32, 0, 0, false, RF_PLAN(float, 2, 4, 16, 8, 4, true, "rf_f32_R2G4_16x8_x4_stage")},
    {BQR_R32, 48, 48, 0, 0, false, RF_PLAN(float, 4, 4, 12, 12, 2, true, "rf_f32_R4G4_12x12_x2_stage")},
    {BQR_R32, 64, 64, 0, 0, false, RF_PLAN(float, 4, 8, 16, 8, 2, true, "rf_f32_R4G8_16x8_x2_stage")},
    {BQR_R32, 80, 80, 0, 0, false, RF_PLAN(float, 8, 8, 10, 10, 1, false, "rf_f32_R8G8_10x10_cta")},
    {BQR_R32, 96, 96, 0, 0, false, RF_PLAN(float, 8, 8, 12, 12, 1, false, "rf_f32_R8G8_12x12_cta")},
    {BQR_R32, 128, 128, 0, 0, false, RF_PLAN(float, 16, 16, 8, 8, 1, false, "rf_f32_R16G16_8x8_cta")},
    {BQR_R32, 256, 64, 0, 0, false, RF_PLAN(float, 32, 8, 8, 8, 1, false, "rf_f32_R32G8_8x8_cta")},
    // complex64 classes
    {BQR_C64, 16, 16, 0, 0, false, RF_PLAN(float2, 2, 2, 8, 8, 8, false, "rf_c64_R2G2_8x8_x8_warp")},
    {BQR_C64, 32, 32, 0, 0, false, RF_PLAN(float2, 4, 4, 8, 8, 2, false, "rf_c64_R4G4_8x8_x2_warp")},
    {BQR_C64, 48, 48, 0, 0, false, RF_PLAN(float2, 8, 8, 6, 6, 1, false, "rf_c64_R8G8_6x6_cta")},
    {BQR_C64, 64, 64, 0, 0, false, RF_PLAN(float2, 8, 8, 8, 8, 1, false, "rf_c64_R8G8_8x8_cta")},
    {BQR_C64, 96, 96, 0, 0, false, RF_PLAN(float2, 16, 16, 6, 6, 1, false, "rf_c64_R16G16_6x6_cta")},
    {BQR_C64, 128, 128, 0, 0, false, RF_PLAN(float2, 16, 16, 8, 8, 1, false, "rf_c64_R16G16_8x8_cta")},
    {BQR_C64, 256, 96, 0, 0, false, RF_PLAN(float2, 32, 16, 8, 6, 1, false, "rf_c64_R32G16_8x6_cta")},
};

const char *forced_variant() {
  static const char *v = std::getenv("BQR_FORCE_VARIANT");
  return (v && *v) ? v : nullptr;
}

const Plan *pick(bqr_dtype_t dt, int m, int n) {
  if (const char *f = forced_variant()) {
    for (const auto &e : kClasses)
      if (e.dt == dt && std::strcmp(e.plan.name, f) == 0 && m <= e.mmax && n <= e.nmax) return &e.plan;
  }
  for (const auto &e : kClasses)
    if (e.dt == dt && !e.alt && e.exact_m == m && e.exact_n == n) return &e.plan;
  for (const auto &e : kClasses)
    if (e.dt == dt && !e.alt && e.exact_m == 0 && m <= e.mmax && n <= e.nmax) return &e.plan;
  return nullptr;
}

// tiny exact sizes 1 <= n <= m <= 8
template <class T, int M>
Plan tiny_plan_n(int n) {
  switch (n) {
#define TN(NN) \
  case NN:     \
    if constexpr (NN <= M) return Plan{"tiny", &launch_tiny<T, M, NN>, nullptr}; break;
    TN(1) TN(2) TN(3) TN(4) TN(5) TN(6) TN(7) TN(8)
#undef TN
  }
  return Plan{nullptr, nullptr, nullptr};
}

template <class T>
Plan tiny_plan(int m, int n) {
  switch (m) {
    case 1: return tiny_plan_n<T, 1>(n);
    case 2: return tiny_plan_n<T, 2>(n);
    case 3: return tiny_plan_n<T, 3>(n);
    case 4: return tiny_plan_n<T, 4>(n);
    case 5: return tiny_plan_n<T, 5>(n);
    case 6: return tiny_plan_n<T, 6>(n);
    case 7: return tiny_plan_n<T, 7>(n);
    case 8: return tiny_plan_n<T, 8>(n);
  }
  return Plan{nullptr, nullptr, nullptr};
}

// fused geqrf + Q^H B: first direct-load class whose tile holds n + nrhs
// columns (the augmented matrix of P:L313)
const Plan *pick_fused(bqr_dtype_t dt, int m, int n, int nrhs) {
  const Plan *best = nullptr;
  int best_area = 1 << 30;
  for (const auto &e : kClasses) {
    if (e.dt != dt || m > e.mmax || n + nrhs > e.nmax) continue;
    if (!std::strstr(e.plan.name, "_aug")) continue;
    const int area = e.mmax * e.nmax;
    if (area < best_area) { best = &e.plan; best_area = area; }
  }
  return best;
}

// Oversize shapes (no single-SM class holds m x n; paper Sec. VII: "a
// sequential tiled QR factorization algorithm similar to the approach in
// the PLASMA library"): right-looking panels of width nb, each
// factored by the register-file kernel of the tall-skinny class and applied
// to the trailing columns by the Q^H B kernel, on panel views of the batch
// (custom batch strides; 2 launches per panel).
bool tiled_panel_width(bqr_dtype_t dt, int m, int n, int *nb) {
  if (m > 256) return false;
  *nb = dt == BQR_R32 ? 64 : 96;  // widest tall class: fp32 256x64, c64 256x96
  return n > *nb;
}

template <class T>
int launch_apply_views(const void *A, int lda, long long sA, const void *tau, long long sT, void *B, int ldb,
                       long long sB, int m, int k, int nrhs, long long batch, cudaStream_t s);

int geqrf_tiled(bqr_dtype_t dt, int m, int n, long long batch, void *A, int lda, void *tau, int nb,
                cudaStream_t stream) {
  const int kmax = std::min(m, n);
  const size_t es = dt == BQR_R32 ? 4 : 8;
  const long long sA = (long long)lda * n;
  char *Ab = reinterpret_cast<char *>(A);
  char *tb = reinterpret_cast<char *>(tau);
  for (int k0 = 0; k0 < kmax; k0 += nb) {
    const int w = std::min(nb, kmax - k0), mp = m - k0;
    const Plan *p = pick(dt, mp, w);
    if (!p) return BQR_ERR_NOT_SUPPORTED;
    Call c{Ab + (k0 + (size_t)k0 * lda) * es, tb + (size_t)k0 * es, batch, mp, w, std::min(mp, w), lda, stream};
    c.strideA = sA;
    c.strideT = kmax;
    int st = p->geqrf(c);
    if (st != BQR_SUCCESS) return st;
    const int nrest = n - k0 - w;
    if (nrest > 0) {
      void *Bv = Ab + (k0 + (size_t)(k0 + w) * lda) * es;
      st = dt == BQR_R32
               ? launch_apply_views<float>(c.A, lda, sA, c.tau, kmax, Bv, lda, sA, mp, std::min(mp, w), nrest, batch, stream)
               : launch_apply_views<float2>(c.A, lda, sA, c.tau, kmax, Bv, lda, sA, mp, std::min(mp, w), nrest, batch,
                                            stream);
      if (st != BQR_SUCCESS) return st;
    }
  }
  return BQR_SUCCESS;
}

// geqrf plan; tiny sizes get their own thread-per-matrix kernel.
bool geqrf_plan(bqr_dtype_t dt, int m, int n, Plan *out) {
  if (m <= 8 && n <= m && !forced_variant()) {
    *out = dt == BQR_R32 ? tiny_plan<float>(m, n) : tiny_plan<float2>(m, n);
    return out->geqrf != nullptr;
  }
  const Plan *p = pick(dt, m, n);
  if (!p) return false;
  *out = *p;
  return true;
}

// orgqr has no thread-per-matrix kernel: tiny shapes use the smallest rf class
bool orgqr_plan(bqr_dtype_t dt, int m, int n, Plan *out) {
  const Plan *p = pick(dt, m, n);
  if (!p) return false;
  *out = *p;
  return true;
}

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

// self-test of the branch-free IEEE helpers (bqr_common.cuh) against the
// CUDA library's sqrt.rn / div.rn on random normal operands spanning the
// exponent range the contract (reading Q6) can produce.
__device__ __forceinline__ unsigned hash32(unsigned x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
  return x;
}
__device__ __forceinline__ float rand_normal_float(unsigned h, int emin, int emax) {
  const unsigned mant = h & 0x7fffffU;
  const int e = emin + (int)((h >> 23) % (unsigned)(emax - emin + 1));
  return __uint_as_float(((unsigned)(e + 127) << 23) | mant);
}
__global__ void selftest_math_kernel(long long n, unsigned seed, unsigned long long *counts) {
  unsigned long long bad_sqrt = 0, bad_div = 0, bad_rcp = 0;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    const unsigned h1 = hash32((unsigned)i * 2654435761U ^ seed), h2 = hash32(h1 ^ 0x9e3779b9U);
    const float x = rand_normal_float(h1, -100, 100);           // sigma / |z|^2 range
    const float a = rand_normal_float(h2, -50, 50) * ((h2 & 1) ? -1.f : 1.f);
    const float b = rand_normal_float(h1 ^ h2, -50, 50) * ((h1 & 2) ? -1.f : 1.f);
    bad_sqrt += __float_as_uint(bqr::sqrt_rn(x)) != __float_as_uint(__fsqrt_rn(x));
    bad_div += __float_as_uint(bqr::div_rn(a, b)) != __float_as_uint(__fdiv_rn(a, b));
    bad_rcp += __float_as_uint(bqr::div_rn(1.0f, b)) != __float_as_uint(__frcp_rn(b));
  }
  atomicAdd(&counts[0], bad_sqrt);
  atomicAdd(&counts[1], bad_div);
  atomicAdd(&counts[2], bad_rcp);
}

template <class T>
int launch_apply_views(const void *A, int lda, long long sA, const void *tau, long long sT, void *B, int ldb,
                       long long sB, int m, int k, int nrhs, long long batch, cudaStream_t s) {
  ApplyArgs a{A, tau, B, batch, lda, 0, m, k, nrhs, ldb, sA, sT, sB};
  return apply_dispatch<T>(a, s);
}

bool valid_dtype(int d) { return d == BQR_R32 || d == BQR_C64; }
size_t elem_size(bqr_dtype_t d) { return d == BQR_R32 ? 4 : 8; }

}  // namespace

extern "C" {

const char *bqr_version(void) { return "bqr 0.1.0 (sm_100a)"; }

const char *bqr_status_string(int status) {
  if (status < 0) return "illegal argument (-i = position of the first bad argument)";
  switch (status) {
    case BQR_SUCCESS: return "success";
    case BQR_ERR_NOT_SUPPORTED: return "shape or dtype not supported by any built size class";
    case BQR_ERR_CUDA: return "CUDA error";
    case BQR_ERR_MISALIGNED: return "misaligned pointer";
  }
  return "unknown status";
}

const char *bqr_qhb_kernel_name(bqr_dtype_t dtype, int m, int n, int nrhs) {
  if (!valid_dtype(dtype) || m <= 0 || n <= 0 || m < n || nrhs <= 0) return "";
  const Plan *p = pick_fused(dtype, m, n, nrhs);
  return p ? p->name : "";
}

const char *bqr_kernel_name(bqr_dtype_t dtype, int m, int n) {
  if (!valid_dtype(dtype) || m <= 0 || n <= 0 || m < n) return "";
  Plan p;
  if (!geqrf_plan(dtype, m, n, &p)) {
    int nb;
    return tiled_panel_width(dtype, m, n, &nb) ? (dtype == BQR_R32 ? "tiled_f32_panel64+apply" : "tiled_c64_panel96+apply")
                                                : "";
  }
  return p.name ? p.name : "";
}

int bqr_geqrf_launches(bqr_dtype_t dtype, int m, int n, int batch) {
  if (!valid_dtype(dtype) || m <= 0 || n <= 0 || batch <= 0 || m < n) return 0;
  Plan p;
  if (geqrf_plan(dtype, m, n, &p)) return 1;
  int nb;
  if (!tiled_panel_width(dtype, m, n, &nb)) return 0;
  int launches = 0;
  const int kmax = std::min(m, n);
  for (int k0 = 0; k0 < kmax; k0 += nb) launches += (n - k0 - std::min(nb, kmax - k0) > 0) ? 2 : 1;
  return launches;
}

int bqr_geqrf_batched(bqr_dtype_t dtype, int m, int n, int batch, void *A, int lda, void *tau,
                      cudaStream_t stream) {
  if (!valid_dtype(dtype)) return -1;
  if (m < 0) return -2;
  if (n < 0) return -3;
  if (batch < 0) return -4;
  const bool work = m > 0 && n > 0 && batch > 0;
  if (work && A == nullptr) return -5;
  if (lda < std::max(1, m)) return -6;
  if (work && tau == nullptr) return -7;
  if (!work) return BQR_SUCCESS;
  if ((reinterpret_cast<uintptr_t>(A) | reinterpret_cast<uintptr_t>(tau)) % elem_size(dtype))
    return BQR_ERR_MISALIGNED;
  if (m < n) return BQR_ERR_NOT_SUPPORTED;
  Plan p;
  if (!geqrf_plan(dtype, m, n, &p)) {
    int nb;
    if (tiled_panel_width(dtype, m, n, &nb)) return geqrf_tiled(dtype, m, n, batch, A, lda, tau, nb, stream);
    return BQR_ERR_NOT_SUPPORTED;
  }
  Call c{A, tau, batch, m, n, std::min(m, n), lda, stream};
  return p.geqrf(c);
}

int bqr_geqrf_qhb_batched(bqr_dtype_t dtype, int m, int n, int nrhs, int batch, void *A, int lda, void *tau,
                          void *B, int ldb, cudaStream_t stream) {
  if (!valid_dtype(dtype)) return -1;
  if (m < 0) return -2;
  if (n < 0) return -3;
  if (nrhs < 0) return -4;
  if (batch < 0) return -5;
  const bool work = m > 0 && n > 0 && batch > 0;
  if (work && A == nullptr) return -6;
  if (lda < std::max(1, m)) return -7;
  if (work && tau == nullptr) return -8;
  if (work && nrhs > 0 && B == nullptr) return -9;
  if (ldb < std::max(1, m)) return -10;
  if (!work) return BQR_SUCCESS;
  if ((reinterpret_cast<uintptr_t>(A) | reinterpret_cast<uintptr_t>(tau) | reinterpret_cast<uintptr_t>(B)) %
      elem_size(dtype))
    return BQR_ERR_MISALIGNED;
  if (m < n) return BQR_ERR_NOT_SUPPORTED;
  const int k = std::min(m, n);
  if (const Plan *p = (nrhs > 0) ? pick_fused(dtype, m, n, nrhs) : nullptr) {
    Call c{A, tau, batch, m, n, k, lda, stream};
    c.B = B;
    c.ldb = ldb;
    c.nrhs = nrhs;
    const int st = p->geqrf(c);
    if (st != BQR_ERR_NOT_SUPPORTED) return st;
  }
  // no class holds the augmented tile: factor, then apply (two launches)
  int st = bqr_geqrf_batched(dtype, m, n, batch, A, lda, tau, stream);
  if (st != BQR_SUCCESS || nrhs == 0) return st;
  return bqr_apply_qh_batched(dtype, m, n, k, nrhs, batch, A, lda, tau, B, ldb, stream);
}

int bqr_orgqr_batched(bqr_dtype_t dtype, int m, int n, int k, int batch, void *A, int lda,
                      const void *tau, cudaStream_t stream) {
  if (!valid_dtype(dtype)) return -1;
  if (m < 0) return -2;
  if (n < 0 || n > m) return -3;
  if (k < 0 || k > n) return -4;
  if (batch < 0) return -5;
  const bool work = m > 0 && n > 0 && batch > 0;
  if (work && A == nullptr) return -6;
  if (lda < std::max(1, m)) return -7;
  if (work && k > 0 && tau == nullptr) return -8;
  if (!work) return BQR_SUCCESS;
  if ((reinterpret_cast<uintptr_t>(A) | reinterpret_cast<uintptr_t>(tau)) % elem_size(dtype))
    return BQR_ERR_MISALIGNED;
  Plan p;
  if (!orgqr_plan(dtype, m, n, &p)) return BQR_ERR_NOT_SUPPORTED;
  Call c{A, const_cast<void *>(tau), batch, m, n, k, lda, stream};
  return p.orgqr(c);
}

int bqr_apply_qh_batched(bqr_dtype_t dtype, int m, int n, int k, int nrhs, int batch, const void *A,
                         int lda, const void *tau, void *B, int ldb, cudaStream_t stream) {
  if (!valid_dtype(dtype)) return -1;
  if (m < 0) return -2;
  if (n < 0) return -3;
  if (k < 0 || k > std::min(m, n)) return -4;
  if (nrhs < 0) return -5;
  if (batch < 0) return -6;
  const bool work = m > 0 && nrhs > 0 && batch > 0;
  if (work && k > 0 && A == nullptr) return -7;
  if (lda < std::max(1, m)) return -8;
  if (work && k > 0 && tau == nullptr) return -9;
  if (work && B == nullptr) return -10;
  if (ldb < std::max(1, m)) return -11;
  if (!work || k == 0) return BQR_SUCCESS;
  if ((reinterpret_cast<uintptr_t>(A) | reinterpret_cast<uintptr_t>(tau) |
       reinterpret_cast<uintptr_t>(B)) % elem_size(dtype))
    return BQR_ERR_MISALIGNED;
  ApplyArgs a{A, tau, B, batch, lda, n, m, k, nrhs, ldb, (long long)lda * n, (long long)k, (long long)ldb * nrhs};
  return dtype == BQR_R32 ? apply_dispatch<float>(a, stream) : apply_dispatch<float2>(a, stream);
}

int bqr_selftest_math(long long n, unsigned seed, unsigned long long *counts, cudaStream_t stream) {
  if (n < 0) return -1;
  if (counts == nullptr) return -3;
  selftest_math_kernel<<<1184, 256, 0, stream>>>(n, seed, counts);
  return finish_launch();
}

size_t bqr_host_workspace_bytes(bqr_dtype_t dtype, int m, int n, int lda, int chunk) {
  if (!valid_dtype(dtype) || m <= 0 || n <= 0 || chunk <= 0) return 0;
  const size_t s = elem_size(dtype);
  const size_t per = ((size_t)lda * n + std::min(m, n)) * s;
  return 2 * per * (size_t)chunk + 256;
}

// Host-buffer streaming: chunks of the batch ping-pong through two device
// buffers; H2D(i+1) overlaps geqrf(i) and D2H(i-1) via two internal streams
// ordered by events.  Synchronous.
int bqr_geqrf_batched_host(bqr_dtype_t dtype, int m, int n, int batch, void *A_host, int lda,
                           void *tau_host, void *workspace, size_t workspace_bytes,
                           cudaStream_t stream) {
  if (!valid_dtype(dtype)) return -1;
  if (m < 0) return -2;
  if (n < 0) return -3;
  if (batch < 0) return -4;
  const bool work = m > 0 && n > 0 && batch > 0;
  if (work && A_host == nullptr) return -5;
  if (lda < std::max(1, m)) return -6;
  if (work && tau_host == nullptr) return -7;
  if (work && workspace == nullptr) return -8;
  if (!work) return BQR_SUCCESS;
  const size_t s = elem_size(dtype);
  const int k = std::min(m, n);
  const size_t mat_bytes = (size_t)lda * n * s, tau_bytes = (size_t)k * s;
  const size_t per = mat_bytes + tau_bytes;
  if (m < n) return BQR_ERR_NOT_SUPPORTED;
  Plan p;
  if (!geqrf_plan(dtype, m, n, &p)) return BQR_ERR_NOT_SUPPORTED;
  auto r256 = [](size_t x) { return (x + 255) & ~size_t(255); };
  auto need = [&](long long ch) { return 2 * (r256(mat_bytes * ch) + r256(tau_bytes * ch)) + 256; };
  long long chunk = std::min<long long>(batch, (long long)(workspace_bytes / (2 * per)));
  while (chunk > 0 && need(chunk) > workspace_bytes) chunk -= std::max<long long>(1, chunk / 64);
  if (chunk < 1) return -9;
  // two buffers [A chunk | tau chunk], 256-byte aligned
  char *ws = reinterpret_cast<char *>((reinterpret_cast<uintptr_t>(workspace) + 255) & ~uintptr_t(255));
  const size_t abytes = r256(mat_bytes * chunk), tbytes = r256(tau_bytes * chunk);
  char *bufA[2] = {ws, ws + abytes + tbytes};
  char *bufT[2] = {ws + abytes, ws + 2 * abytes + tbytes};
  cudaStream_t st[3] = {stream, nullptr, nullptr};  // compute, h2d, d2h
  cudaEvent_t ev_in[2], ev_done[2], ev_out[2];
  int status = BQR_SUCCESS;
  if (cudaStreamCreateWithFlags(&st[1], cudaStreamNonBlocking) != cudaSuccess ||
      cudaStreamCreateWithFlags(&st[2], cudaStreamNonBlocking) != cudaSuccess)
    return BQR_ERR_CUDA;
  for (int i = 0; i < 2; ++i) {
    cudaEventCreateWithFlags(&ev_in[i], cudaEventDisableTiming);
    cudaEventCreateWithFlags(&ev_done[i], cudaEventDisableTiming);
    cudaEventCreateWithFlags(&ev_out[i], cudaEventDisableTiming);
  }
  // order the copies after whatever the caller already queued on `stream`
  cudaEvent_t ev_entry;
  cudaEventCreateWithFlags(&ev_entry, cudaEventDisableTiming);
  cudaEventRecord(ev_entry, st[0]);
  cudaStreamWaitEvent(st[1], ev_entry, 0);
  cudaEventDestroy(ev_entry);
  const long long nchunks = (batch + chunk - 1) / chunk;
  bool out_pending[2] = {false, false};
  for (long long ci = 0; ci < nchunks && status == BQR_SUCCESS; ++ci) {
    const int b = (int)(ci & 1);
    const long long b0 = ci * chunk;
    const long long cnt = std::min<long long>(chunk, batch - b0);
    // buffer b free once its previous D2H finished
    if (out_pending[b]) cudaStreamWaitEvent(st[1], ev_out[b], 0);
    cudaMemcpyAsync(bufA[b], reinterpret_cast<char *>(A_host) + b0 * mat_bytes, cnt * mat_bytes,
                    cudaMemcpyHostToDevice, st[1]);
    cudaEventRecord(ev_in[b], st[1]);
    cudaStreamWaitEvent(st[0], ev_in[b], 0);
    Call c{bufA[b], bufT[b], cnt, m, n, k, lda, st[0]};
    status = p.geqrf(c);
    cudaEventRecord(ev_done[b], st[0]);
    cudaStreamWaitEvent(st[2], ev_done[b], 0);
    cudaMemcpyAsync(reinterpret_cast<char *>(A_host) + b0 * mat_bytes, bufA[b], cnt * mat_bytes,
                    cudaMemcpyDeviceToHost, st[2]);
    cudaMemcpyAsync(reinterpret_cast<char *>(tau_host) + b0 * tau_bytes, bufT[b], cnt * tau_bytes,
                    cudaMemcpyDeviceToHost, st[2]);
    cudaEventRecord(ev_out[b], st[2]);
    out_pending[b] = true;
  }
  if (cudaStreamSynchronize(st[2]) != cudaSuccess || cudaStreamSynchronize(st[0]) != cudaSuccess)
    status = BQR_ERR_CUDA;
  for (int i = 0; i < 2; ++i) {
    cudaEventDestroy(ev_in[i]);
    cudaEventDestroy(ev_done[i]);
    cudaEventDestroy(ev_out[i]);
  }
  cudaStreamDestroy(st[1]);
  cudaStreamDestroy(st[2]);
  if (status == BQR_SUCCESS && cudaGetLastError() != cudaSuccess) status = BQR_ERR_CUDA;
  return status;
}

}  // extern "C"

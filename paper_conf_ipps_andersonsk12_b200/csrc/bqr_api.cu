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

#include "bqr_launch.cuh"

namespace bqr {
namespace host {

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

}  // namespace host
}  // namespace bqr

namespace {

using namespace bqr;
using namespace bqr::host;

// All size classes, in dispatch order: headline exact shapes and augmented
// classes, then fp32, then complex64, then the
// experiment-only alternatives (BQR_FORCE_VARIANT).
struct Tables {
  static constexpr int kN = 8;
  const ClassEntry *t[kN];
  int n[kN];
  Tables() {
    t[0] = classes_ll(&n[0]);
    t[1] = classes_llc(&n[1]);
    t[2] = classes_co(&n[2]);
    t[3] = classes_headline(&n[3]);
    t[4] = classes_f32(&n[4]);
    t[5] = classes_c64(&n[5]);
    t[6] = classes_alt(&n[6]);
    t[7] = classes_cl(&n[7]);
  }
  template <class F>
  const Plan *find(F pred) const {
    for (int a = 0; a < kN; ++a)
      for (int i = 0; i < n[a]; ++i)
        if (pred(t[a][i])) return &t[a][i].plan;
    return nullptr;
  }
  template <class F>
  void each(F f) const {
    for (int a = 0; a < kN; ++a)
      for (int i = 0; i < n[a]; ++i) f(t[a][i]);
  }
};

const Tables &tables() {
  static const Tables tb;
  return tb;
}

const char *forced_variant() {
  static const char *v = std::getenv("BQR_FORCE_VARIANT");
  return (v && *v) ? v : nullptr;
}

const Plan *pick(bqr_dtype_t dt, int m, int n) {
  const Tables &tb = tables();
  if (const char *f = forced_variant()) {
    if (const Plan *p = tb.find([&](const ClassEntry &e) {
          return e.dt == dt && std::strcmp(e.plan.name, f) == 0 && m <= e.mmax && n <= e.nmax;
        }))
      return p;
  }
  if (const Plan *p = tb.find([&](const ClassEntry &e) {
        return e.dt == dt && !e.alt && e.exact_m == m && e.exact_n == n;
      }))
    return p;
  return tb.find([&](const ClassEntry &e) {
    return e.dt == dt && !e.alt && e.exact_m == 0 && m <= e.mmax && n <= e.nmax;
  });
}

// fused geqrf + Q^H B: smallest augmented class whose tile holds n + nrhs
// columns (the augmented matrix of P:L313)
const Plan *pick_fused(bqr_dtype_t dt, int m, int n, int nrhs) {
  if (const char *f = forced_variant()) {
    if (const Plan *p = tables().find([&](const ClassEntry &e) {
          return e.dt == dt && std::strcmp(e.plan.name, f) == 0 && std::strstr(f, "_aug") && m <= e.mmax &&
                 n + nrhs <= e.nmax;
        }))
      return p;
  }
  const Plan *best = nullptr;
  int best_area = 1 << 30;
  tables().each([&](const ClassEntry &e) {
    if (e.dt != dt || m > e.mmax || n + nrhs > e.nmax) return;
    if (std::strncmp(e.plan.name, "alt_", 4) == 0) return;  // experiment-only variants (BQR_FORCE_VARIANT)
    if (!std::strstr(e.plan.name, "_aug")) return;
    // exact-shape fused classes (bounds == exact shape) only for that shape
    if (e.exact_m > 0 && e.mmax == e.exact_m && e.nmax == e.exact_n && (e.exact_m != m || e.exact_n != n + nrhs))
      return;
    const int area = e.mmax * e.nmax;
    if (area < best_area) {
      best = &e.plan;
      best_area = area;
    }
  });
  return best;
}

int apply_dispatch_t(bqr_dtype_t dt, const ApplyArgs &a, cudaStream_t s) {
  return dt == BQR_R32 ? apply_dispatch_f32(a, s) : apply_dispatch_c64(a, s);
}

// Oversize shapes (no single-SM class holds m x n; paper Sec. VII: "a
// sequential tiled QR factorization algorithm similar to the approach in
// the PLASMA library"): right-looking panels of width nb, each
// factored by the register-file kernel of the tall-skinny class and applied
// to the trailing columns by the Q^H B kernel, on panel views of the batch
// (custom batch strides; 2 launches per panel).
bool tiled_panel_width(bqr_dtype_t dt, int m, int n, int *nb) {
  // fp32 up to 256 x 256 always has a single-SM class (bqr_classes_f32.cu),
  // so only complex shapes beyond 160 x 160 take the tiled path
  if (m > 256 || dt != BQR_C64) return false;
  *nb = 96;  // widest tall complex class: 256 x 96
  return n > *nb;
}

// compact-WY blocked variant (bqr_wy.cu): register-file panels (64 fp32 /
// 96 complex columns) + tensor-core trailing updates
const Plan *pick_c64_panel(int m, int n) { return pick(BQR_C64, m, n); }
const Plan *pick_f32_panel(int m, int n) { return pick(BQR_R32, m, n); }
constexpr size_t kWyMaxWorkspace = size_t(2) << 30;  // stream-ordered workspace cap of the default path

const char *wy_name(bqr_dtype_t dt) {
  return dt == BQR_R32 ? "wy_f32_panel64+tcgen05_fastf32_gemm" : "wy_c64_panel96+tcgen05_fastf32_gemm";
}

// shapes bqr_geqrf_batched itself factors with the blocked variant: the
// complex ones beyond every single-SM class (measured 1.4-1.8x faster than
// the tiled panels, profiles/r02/experiments/wy_vs_tiled.jsonl)
bool wy_default_shape(bqr_dtype_t dt, int m, int n, int lda) {
  return dt == BQR_C64 && n > 160 && wy_supported(dt, m, n, lda) && !forced_variant();
}

bool wy_default(bqr_dtype_t dt, int m, int n, int lda, const void *A) {
  return wy_default_shape(dt, m, n, lda) && (reinterpret_cast<uintptr_t>(A) & 15) == 0;
}

// a library-private stream-ordered memory pool per device that keeps its
// memory between calls (release threshold: unlimited), so repeated calls do
// not remap the workspace; created once, like the kernel attributes
cudaMemPool_t wy_pool() {
  static cudaMemPool_t pools[kMaxDevices] = {};
  static std::once_flag once[kMaxDevices];
  const int d = current_device();
  std::call_once(once[d], [d] {
    cudaMemPoolProps props = {};
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = d;
    cudaMemPool_t p = nullptr;
    if (cudaMemPoolCreate(&p, &props) == cudaSuccess) {
      unsigned long long thr = ~0ULL;
      cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &thr);
      pools[d] = p;
    } else {
      cudaGetLastError();
    }
  });
  return pools[d];
}

// bqr_geqrf_batched's path for those shapes: the blocked variant on a
// workspace taken from the library's stream-ordered memory pool on the
// caller's stream (cudaMallocFromPoolAsync / cudaFreeAsync: no host
// synchronisation, private to this call); the tiled path if the pool cannot
// provide it
int geqrf_wy_default(bqr_dtype_t dt, int m, int n, long long batch, void *A, int lda, void *tau,
                     cudaStream_t stream) {
  const size_t per = wy_workspace_bytes(dt, m, n, 1);
  const long long chunk = std::max<long long>(1, std::min<long long>(batch, (long long)(kWyMaxWorkspace / per)));
  const size_t bytes = wy_workspace_bytes(dt, m, n, (int)chunk);
  cudaMemPool_t pool = wy_pool();
  void *ws = nullptr;
  if (!pool || cudaMallocFromPoolAsync(&ws, bytes, pool, stream) != cudaSuccess) {
    cudaGetLastError();
    return BQR_ERR_NOT_SUPPORTED;
  }
  const int st = geqrf_wy(dt, m, n, batch, A, lda, tau, ws, bytes, stream,
                          dt == BQR_R32 ? &pick_f32_panel : &pick_c64_panel);
  cudaFreeAsync(ws, stream);
  return st;
}

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
      ApplyArgs a{c.A, c.tau, Bv, batch, lda, 0, mp, std::min(mp, w), nrest, lda, sA, (long long)kmax, sA};
      st = apply_dispatch_t(dt, a, stream);
      if (st != BQR_SUCCESS) return st;
    }
  }
  return BQR_SUCCESS;
}

// geqrf plan; tiny sizes get their own thread-per-matrix kernel.
bool geqrf_plan(bqr_dtype_t dt, int m, int n, Plan *out) {
  if (m <= 8 && n <= m && !forced_variant()) {
    *out = dt == BQR_R32 ? tiny_plan_f32(m, n) : tiny_plan_c64(m, n);
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

bool valid_dtype(int d) { return d == BQR_R32 || d == BQR_C64; }
size_t elem_size(bqr_dtype_t d) { return d == BQR_R32 ? 4 : 8; }

}  // namespace

// ---- host-buffer pipeline state: two copy streams and the events of a
// kHostRing-buffer rotation, created once per device (never destroyed;
// like the kernel attributes) so a call does not pay stream creation
constexpr int kHostRing = 3;
struct HostPipe {
  std::mutex mu;  // one host call at a time per device: the events and copy streams are shared
  cudaStream_t h2d = nullptr, d2h = nullptr;
  cudaEvent_t entry = nullptr, in[kHostRing] = {}, done[kHostRing] = {}, out[kHostRing] = {};
  bool ok = false;
};

static HostPipe *host_pipe() {
  static HostPipe pipes[bqr::host::kMaxDevices];
  static std::once_flag once[bqr::host::kMaxDevices];
  const int d = bqr::host::current_device();
  std::call_once(once[d], [d] {
    HostPipe &h = pipes[d];
    bool ok = cudaStreamCreateWithFlags(&h.h2d, cudaStreamNonBlocking) == cudaSuccess &&
              cudaStreamCreateWithFlags(&h.d2h, cudaStreamNonBlocking) == cudaSuccess &&
              cudaEventCreateWithFlags(&h.entry, cudaEventDisableTiming) == cudaSuccess;
    for (int i = 0; i < kHostRing && ok; ++i)
      ok = cudaEventCreateWithFlags(&h.in[i], cudaEventDisableTiming) == cudaSuccess &&
           cudaEventCreateWithFlags(&h.done[i], cudaEventDisableTiming) == cudaSuccess &&
           cudaEventCreateWithFlags(&h.out[i], cudaEventDisableTiming) == cudaSuccess;
    h.ok = ok;
  });
  return pipes[d].ok ? &pipes[d] : nullptr;
}

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
    if (!tiled_panel_width(dtype, m, n, &nb)) return "";
    return wy_default_shape(dtype, m, n, m) ? wy_name(dtype) : "tiled_c64_panel96+apply";
  }
  return p.name ? p.name : "";
}

long long bqr_resident_matrices(bqr_dtype_t dtype, int m, int n) {
  if (!valid_dtype(dtype) || m <= 0 || n <= 0 || m < n) return 0;
  Plan p;
  if (!geqrf_plan(dtype, m, n, &p)) return 0;  // tiled oversize path: several launches
  long long r = 0;
  Call c{nullptr, nullptr, 1, m, n, std::min(m, n), m, nullptr};
  c.resident = &r;
  return p.geqrf(c) == BQR_SUCCESS ? r : 0;
}

// ---- compact-WY blocked variant (bqr_wy.cu): explicit workspace entry point

size_t bqr_geqrf_wy_workspace_bytes(bqr_dtype_t dtype, int m, int n, int lda, int chunk) {
  if (!valid_dtype(dtype) || m <= 0 || n <= 0 || chunk <= 0) return 0;
  if (!wy_supported(dtype, m, n, lda)) return 0;
  return wy_workspace_bytes(dtype, m, n, chunk);
}

const char *bqr_geqrf_wy_kernel_name(bqr_dtype_t dtype, int m, int n, int lda) {
  if (!valid_dtype(dtype) || m <= 0 || n <= 0 || m < n) return "";
  if (!wy_supported(dtype, m, n, lda)) return bqr_kernel_name(dtype, m, n);
  return wy_name(dtype);
}

int bqr_geqrf_wy_batched(bqr_dtype_t dtype, int m, int n, int batch, void *A, int lda, void *tau, void *work,
                         size_t work_bytes, cudaStream_t stream) {
  if (!valid_dtype(dtype)) return -1;
  if (m < 0) return -2;
  if (n < 0) return -3;
  if (batch < 0) return -4;
  const bool work_needed = m > 0 && n > 0 && batch > 0;
  if (work_needed && A == nullptr) return -5;
  if (lda < std::max(1, m)) return -6;
  if (work_needed && tau == nullptr) return -7;
  if (!work_needed) return BQR_SUCCESS;
  if (!wy_supported(dtype, m, n, lda) || (reinterpret_cast<uintptr_t>(A) & 15))
    return bqr_geqrf_batched(dtype, m, n, batch, A, lda, tau, stream);  // no blocked variant for this shape
  if (work == nullptr) return -8;
  if (work_bytes < wy_workspace_bytes(dtype, m, n, 1)) return -9;
  return geqrf_wy(dtype, m, n, batch, A, lda, tau, work, work_bytes, stream,
                  dtype == BQR_R32 ? &pick_f32_panel : &pick_c64_panel);
}

int bqr_class_count(void) {
  int total = 0;
  tables().each([&](const ClassEntry &) { ++total; });
  return total;
}

const char *bqr_class_info(int index, int *dtype, int *mmax, int *nmax, int *exact_m, int *exact_n, int *flags) {
  if (index < 0) return nullptr;
  const ClassEntry *found = nullptr;
  int i = 0;
  tables().each([&](const ClassEntry &e) {
    if (i++ == index) found = &e;
  });
  if (!found) return nullptr;
  if (dtype) *dtype = found->dt;
  if (mmax) *mmax = found->mmax;
  if (nmax) *nmax = found->nmax;
  if (exact_m) *exact_m = found->exact_m;
  if (exact_n) *exact_n = found->exact_n;
  const bool aug = std::strstr(found->plan.name, "_aug") != nullptr;
  const bool experiment = std::strncmp(found->plan.name, "alt_", 4) == 0;
  if (flags) *flags = (experiment ? 1 : 0) | (aug ? 2 : 0) | (found->alt ? 4 : 0);
  return found->plan.name;
}

int bqr_geqrf_launches(bqr_dtype_t dtype, int m, int n, int batch) {
  if (!valid_dtype(dtype) || m <= 0 || n <= 0 || batch <= 0 || m < n) return 0;
  Plan p;
  if (geqrf_plan(dtype, m, n, &p)) return 1;
  int nb;
  if (!tiled_panel_width(dtype, m, n, &nb)) return 0;
  const bool wy = wy_default_shape(dtype, m, n, m);
  const int kmax = std::min(m, n);
  // per panel: tiled = panel + apply; WY = panel + V extraction + 4 GEMMs + xLARFT
  // + the accumulate C += D
  // (one chunk when the batch fits the default path's workspace)
  const long long per_chunk =
      wy ? std::max<long long>(1, (long long)(kWyMaxWorkspace / wy_workspace_bytes(dtype, m, n, 1))) : batch;
  const long long chunks = (batch + per_chunk - 1) / per_chunk;
  int launches = 0;
  for (int k0 = 0; k0 < kmax; k0 += nb)
    launches += (n - k0 - std::min(nb, kmax - k0) > 0) ? (wy ? 8 : 2) : 1;
  return (int)(launches * chunks);
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
    if (!tiled_panel_width(dtype, m, n, &nb)) return BQR_ERR_NOT_SUPPORTED;
    if (wy_default(dtype, m, n, lda, A) && !forced_variant()) {
      const int st = geqrf_wy_default(dtype, m, n, batch, A, lda, tau, stream);
      if (st != BQR_ERR_NOT_SUPPORTED) return st;
    }
    return geqrf_tiled(dtype, m, n, batch, A, lda, tau, nb, stream);
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

int bqr_gels_batched(bqr_dtype_t dtype, int m, int n, int nrhs, int batch, void *A, int lda, void *tau, void *B,
                     int ldb, int *info, cudaStream_t stream) {
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
  if (m < n) return BQR_ERR_NOT_SUPPORTED;  // minimum-norm (underdetermined) problems are not built
  if (n > 256) return BQR_ERR_NOT_SUPPORTED;
  if ((reinterpret_cast<uintptr_t>(A) | reinterpret_cast<uintptr_t>(tau) | reinterpret_cast<uintptr_t>(B)) %
      elem_size(dtype))
    return BQR_ERR_MISALIGNED;
  // factor [A | B] (Q^H B falls out of the factorisation) ...
  int st = bqr_geqrf_qhb_batched(dtype, m, n, nrhs, batch, A, lda, tau, B, ldb, stream);
  if (st != BQR_SUCCESS) return st;
  // ... then the triangular system by row operations
  return solve_upper_dispatch(dtype, A, lda, (long long)lda * n, B, ldb, (long long)ldb * nrhs, info, batch, n,
                              nrhs, stream);
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
  if (!orgqr_plan(dtype, m, n, &p)) {
    // beyond the single-SM classes (complex > 160): xORGQR by 96-column
    // compact-WY panels on the tensor cores, workspace from the private pool
    if (!wy_supported(dtype, m, n, lda) || (reinterpret_cast<uintptr_t>(A) & 15))
      return BQR_ERR_NOT_SUPPORTED;
    const size_t per = orgqr_wy_workspace_bytes(dtype, m, n, k, 1);
    const long long chunk = std::max<long long>(1, std::min<long long>(batch, (long long)(kWyMaxWorkspace / per)));
    const size_t bytes = orgqr_wy_workspace_bytes(dtype, m, n, k, (int)chunk);
    cudaMemPool_t pool = wy_pool();
    void *ws = nullptr;
    if (!pool || cudaMallocFromPoolAsync(&ws, bytes, pool, stream) != cudaSuccess) {
      cudaGetLastError();
      return BQR_ERR_CUDA;
    }
    const int st = orgqr_wy(dtype, m, n, k, batch, A, lda, tau, ws, bytes, stream);
    cudaFreeAsync(ws, stream);
    return st;
  }
  Call c{A, const_cast<void *>(tau), batch, m, n, k, lda, stream};
  c.strideT = n;  // tau batch stride min(m, n) = n, as bqr_geqrf_batched wrote it
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
  // tau batch stride min(m, n): the stride bqr_geqrf_batched wrote, also when k < min(m, n)
  ApplyArgs a{A, tau, B, batch, lda, n, m, k, nrhs, ldb, (long long)lda * n, (long long)std::min(m, n),
              (long long)ldb * nrhs};
  return apply_dispatch_t(dtype, a, stream);
}

int bqr_selftest_math(long long n, unsigned seed, unsigned long long *counts, cudaStream_t stream) {
  if (n < 0) return -1;
  if (counts == nullptr) return -3;
  return launch_selftest_math(n, seed, counts, stream);
}

size_t bqr_host_workspace_bytes(bqr_dtype_t dtype, int m, int n, int lda, int chunk) {
  if (!valid_dtype(dtype) || m <= 0 || n <= 0 || chunk <= 0) return 0;
  const size_t s = elem_size(dtype);
  const size_t per = ((size_t)lda * n + std::min(m, n)) * s;
  return kHostRing * (per * (size_t)chunk + 512) + 256;
}

// Host-buffer streaming: chunks of the batch rotate through kHostRing device
// buffers; H2D(i+2), geqrf(i+1) and D2H(i) overlap on two internal streams
// (created once per device, like the kernel attributes) ordered by events.
// Synchronous.
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
  constexpr int NB = kHostRing;
  auto r256 = [](size_t x) { return (x + 255) & ~size_t(255); };
  auto need = [&](long long ch) { return NB * (r256(mat_bytes * ch) + r256(tau_bytes * ch)) + 256; };
  long long chunk = std::min<long long>(batch, (long long)(workspace_bytes / (NB * per)));
  while (chunk > 0 && need(chunk) > workspace_bytes) chunk -= std::max<long long>(1, chunk / 64);
  if (chunk < 1) return -9;
  // NB buffers [A chunk | tau chunk], 256-byte aligned
  char *ws = reinterpret_cast<char *>((reinterpret_cast<uintptr_t>(workspace) + 255) & ~uintptr_t(255));
  const size_t abytes = r256(mat_bytes * chunk), tbytes = r256(tau_bytes * chunk);
  char *bufA[NB], *bufT[NB];
  for (int i = 0; i < NB; ++i) {
    bufA[i] = ws + i * (abytes + tbytes);
    bufT[i] = bufA[i] + abytes;
  }
  HostPipe *hp = host_pipe();
  if (!hp) return BQR_ERR_CUDA;
  // re-entrancy: concurrent host calls on one device are serialised (the
  // call is synchronous anyway); without the lock thread B could re-record
  // done[b] between thread A's record and wait, and A's D2H would copy back
  // before its own kernel ran
  std::lock_guard<std::mutex> lock(hp->mu);
  cudaStream_t st[3] = {stream, hp->h2d, hp->d2h};  // compute, h2d, d2h
  int status = BQR_SUCCESS;
  // order the copies after whatever the caller already queued on `stream`
  cudaEventRecord(hp->entry, st[0]);
  cudaStreamWaitEvent(st[1], hp->entry, 0);
  const long long nchunks = (batch + chunk - 1) / chunk;
  bool out_pending[NB] = {};
  for (long long ci = 0; ci < nchunks && status == BQR_SUCCESS; ++ci) {
    const int b = (int)(ci % NB);
    const long long b0 = ci * chunk;
    const long long cnt = std::min<long long>(chunk, batch - b0);
    // buffer b free once its previous D2H finished
    if (out_pending[b]) cudaStreamWaitEvent(st[1], hp->out[b], 0);
    cudaMemcpyAsync(bufA[b], reinterpret_cast<char *>(A_host) + b0 * mat_bytes, cnt * mat_bytes,
                    cudaMemcpyHostToDevice, st[1]);
    cudaEventRecord(hp->in[b], st[1]);
    cudaStreamWaitEvent(st[0], hp->in[b], 0);
    Call c{bufA[b], bufT[b], cnt, m, n, k, lda, st[0]};
    status = p.geqrf(c);
    cudaEventRecord(hp->done[b], st[0]);
    cudaStreamWaitEvent(st[2], hp->done[b], 0);
    cudaMemcpyAsync(reinterpret_cast<char *>(A_host) + b0 * mat_bytes, bufA[b], cnt * mat_bytes,
                    cudaMemcpyDeviceToHost, st[2]);
    cudaMemcpyAsync(reinterpret_cast<char *>(tau_host) + b0 * tau_bytes, bufT[b], cnt * tau_bytes,
                    cudaMemcpyDeviceToHost, st[2]);
    cudaEventRecord(hp->out[b], st[2]);
    out_pending[b] = true;
  }
  if (cudaStreamSynchronize(st[2]) != cudaSuccess || cudaStreamSynchronize(st[0]) != cudaSuccess)
    status = BQR_ERR_CUDA;
  if (status == BQR_SUCCESS && cudaGetLastError() != cudaSuccess) status = BQR_ERR_CUDA;
  return status;
}

}  // extern "C"

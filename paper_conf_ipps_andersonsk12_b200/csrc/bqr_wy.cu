// bqr_wy.cu -- compact-WY blocked QR for matrices beyond one panel
// (north-star "compact-WY blocked variant"; the paper's
// tiled QR for STAP sizes that do not fit one block, and its
// "panel" / blocked algorithms).
//
// Right-looking panels of nb columns:
//   1. the panel A[k0:m, k0:k0+nb] is factored in registers by the
//      single-SM class of its tall-skinny shape (unblocked Householder,
//      bqr_rf.cuh), which leaves V and tau in place (LAPACK storage);
//   2. V (unit lower trapezoidal, m_p x nb) and conj(V) are extracted into
//      the workspace; G = V^H V (a GEMM) and the compact-WY factor T with
//      H_0 ... H_{nb-1} = I - V T V^H (xLARFT recurrence, one CTA per matrix)
//      give Th = T^H;
//   3. the trailing update C <- Q^H C = C - V (T^H (V^H C)) is three batched
//      GEMMs: W = V^H C, X = Th W, C = C - V X.
// The GEMMs are a dense contraction, so they run on the 5th-generation
// tensor cores (tcgen05, SASS UTCHMMA) through CUTLASS's SM100 "FastF32"
// collective, which splits each fp32 operand into bf16 parts and sums the
// partial products in fp32 (fp32-level accuracy: tools/micro/wy_gemm_probe.cu
// measured |error| / (|ref| sqrt K) ~ 2e-8 on these shapes); the panels stay
// on the FP32 CUDA cores with IEEE sqrt/div.
//
// Complex64 (panels of 96) and fp32 (panels of 64, the widest tall
// single-SM classes).  The workspace is caller-owned device memory
// (bqr_geqrf_wy_batched) or comes from a library-private stream-ordered pool
// (bqr_geqrf_batched); the batch is processed in chunks that fit it.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>

#include "bqr_launch.cuh"

#ifdef BQR_NO_CUTLASS
namespace bqr {
namespace host {
int wy_panel_width(bqr_dtype_t dt) { return dt == BQR_R32 ? 64 : 96; }
bool wy_supported(bqr_dtype_t, int, int, int) { return false; }
size_t wy_workspace_bytes(bqr_dtype_t, int, int, int) { return 0; }
int geqrf_wy(bqr_dtype_t, int, int, long long, void *, int, void *, void *, size_t, cudaStream_t,
             const Plan *(*)(int, int)) {
  return BQR_ERR_NOT_SUPPORTED;
}
size_t orgqr_wy_workspace_bytes(bqr_dtype_t, int, int, int, int) { return 0; }
int orgqr_wy(bqr_dtype_t, int, int, int, long long, void *, int, const void *, void *, size_t, cudaStream_t) {
  return BQR_ERR_NOT_SUPPORTED;
}
}  // namespace host
}  // namespace bqr
#else

#include "cutlass/cutlass.h"
#include "cute/tensor.hpp"
#include "cutlass/complex.h"
#include "cutlass/gemm/dispatch_policy.hpp"
#include "cutlass/gemm/collective/collective_builder.hpp"
#include "cutlass/epilogue/collective/collective_builder.hpp"
#include "cutlass/gemm/kernel/gemm_universal.hpp"
#include "cutlass/gemm/device/gemm_universal_adapter.h"

namespace bqr {
namespace wy {

// element traits: the device element (float / float2 interleaved complex)
// and CUTLASS's view of it; TMA rows need 16-byte multiples
template <class E> struct Tr;
template <> struct Tr<float2> {
  using CE = cutlass::complex<float>;
  static constexpr int kAlign = 2;
  static __host__ __device__ CE one() { return CE(1.f, 0.f); }
  static __host__ __device__ CE zero() { return CE(0.f, 0.f); }
  static __host__ __device__ CE mone() { return CE(-1.f, 0.f); }
};
template <> struct Tr<float> {
  using CE = float;
  static constexpr int kAlign = 4;
  static __host__ __device__ CE one() { return 1.f; }
  static __host__ __device__ CE zero() { return 0.f; }
  static __host__ __device__ CE mone() { return -1.f; }
};

// batched GEMM D = alpha A B + beta C on tcgen05 (FastF32 emulation)
template <class E, class LayoutA>
struct Gemm {
  using CE = typename Tr<E>::CE;
  static constexpr int AL = Tr<E>::kAlign;
  using LayoutB = cutlass::layout::ColumnMajor;
  using LayoutC = cutlass::layout::ColumnMajor;
  using MmaTileShape = cute::Shape<cute::_128, cute::_64, cute::_16>;
  using ClusterShape = cute::Shape<cute::_1, cute::_1, cute::_1>;
  using Epi = typename cutlass::epilogue::collective::CollectiveBuilder<
      cutlass::arch::Sm100, cutlass::arch::OpClassTensorOp, MmaTileShape, ClusterShape,
      cutlass::epilogue::collective::EpilogueTileAuto, CE, CE, CE, LayoutC, AL, CE, LayoutC, AL,
      cutlass::epilogue::FastF32NoSmemWarpSpecialized1Sm>::CollectiveOp;
  using Main = typename cutlass::gemm::collective::CollectiveBuilder<
      cutlass::arch::Sm100, cutlass::arch::OpClassTensorOp, CE, LayoutA, AL, CE, LayoutB, AL, CE, MmaTileShape,
      ClusterShape,
      cutlass::gemm::collective::StageCountAutoCarveout<static_cast<int>(sizeof(typename Epi::SharedStorage))>,
      cutlass::gemm::KernelTmaWarpSpecialized1SmFastFP32Sm100>::CollectiveOp;
  using Kernel = cutlass::gemm::kernel::GemmUniversal<cute::Shape<int, int, int, int>, Main, Epi>;
  using Op = cutlass::gemm::device::GemmUniversalAdapter<Kernel>;

  // A: M x K (row-major: element (i, k) at i*lda + k; column-major: i + k*lda),
  // B: K x N column-major, C/D: M x N column-major; per-matrix strides s*.
  static int run(int M, int N, int K, int L, const E *A, int64_t lda, int64_t sA, const E *B, int64_t ldb, int64_t sB,
                 E *C, int64_t ldc, int64_t sC, CE alpha, CE beta, cudaStream_t stream) {
    typename Kernel::StrideA stA;
    if constexpr (cute::is_same_v<LayoutA, cutlass::layout::RowMajor>)
      stA = cute::make_stride(lda, cute::Int<1>{}, sA);
    else
      stA = cute::make_stride(cute::Int<1>{}, lda, sA);
    const typename Kernel::StrideB stB = cute::make_stride(ldb, cute::Int<1>{}, sB);
    const typename Kernel::StrideC stC = cute::make_stride(cute::Int<1>{}, ldc, sC);
    typename Op::Arguments args{cutlass::gemm::GemmUniversalMode::kGemm,
                                {M, N, K, L},
                                {reinterpret_cast<const CE *>(A), stA, reinterpret_cast<const CE *>(B), stB},
                                {{alpha, beta}, reinterpret_cast<CE *>(C), stC, reinterpret_cast<CE *>(C), stC}};
    Op op;
    if (Op::get_workspace_size(args) != 0) return BQR_ERR_NOT_SUPPORTED;  // data-parallel tiles need none
    if (op.can_implement(args) != cutlass::Status::kSuccess) return BQR_ERR_NOT_SUPPORTED;
    if (op.initialize(args, nullptr, stream) != cutlass::Status::kSuccess) return BQR_ERR_CUDA;
    if (op.run(stream) != cutlass::Status::kSuccess) return BQR_ERR_CUDA;
    return cudaGetLastError() == cudaSuccess ? BQR_SUCCESS : BQR_ERR_CUDA;
  }
};

// V (m_p x nb, unit lower trapezoidal) of each matrix's panel and, for
// complex data, conj(V) (the K-major A operand of V^H X)
template <class E>
__global__ void extract_v_kernel(const E *A, long long sA, int lda, int k0, int mp, int nb, long long L, E *V, E *Vc,
                                 int nvalid = 1 << 30) {
  using X = El<E>;
  const long long per = (long long)mp * nb;
  for (long long idx = blockIdx.x * (long long)blockDim.x + threadIdx.x; idx < per * L;
       idx += (long long)gridDim.x * blockDim.x) {
    const long long b = idx / per;
    const int rem = (int)(idx - b * per);
    const int i = rem / mp, r = rem - i * mp;  // column i, row r
    E v = r == i && i < nvalid ? X::one() : X::zero();  // columns >= nvalid: zero padding
    if (r > i && i < nvalid) v = A[b * sA + (long long)(k0 + i) * lda + (k0 + r)];
    V[idx] = v;
    if constexpr (X::kComplex) Vc[idx] = X::conj(v);
  }
}

// sum += a * b (no conjugation)
__device__ __forceinline__ void mac(float2 &s, float2 a, float2 b) {
  s.x = fmaf(a.x, b.x, fmaf(-a.y, b.y, s.x));
  s.y = fmaf(a.x, b.y, fmaf(a.y, b.x, s.y));
}
__device__ __forceinline__ void mac(float &s, float a, float b) { s = fmaf(a, b, s); }

// xLARFT (forward, columnwise): T upper triangular with H_0 ... H_{nb-1} =
// I - V T V^H, from G = V^H V and tau, blocked for parallelism: the 16 x 16
// diagonal blocks by the column recurrence T(i, i) = tau_i,
// T(j, i) = -tau_i sum_{j <= l < i} T(j, l) G(l, i) (one warp each), then
// block column by block column T(0:J, J) = -T(0:J, 0:J) G(0:J, J) T(J, J)
// (the product of two compact-WY factors [V1 V2]: T12 = -T11 V1^H V2 T22).
// Writes Th = T^H (nb x nb, column-major).  One CTA per matrix.
constexpr int kTB = 16;
template <class E>
__global__ void __launch_bounds__(256) larft_kernel(const E *G, const E *tau, long long sTau, int nb, E *Th,
                                                    bool herm = true, int nvalid = 1 << 30) {
  using X = El<E>;
  extern __shared__ __align__(16) unsigned char tsm_raw[];
  E *T = reinterpret_cast<E *>(tsm_raw);  // nb x nb column-major, then P (nb x kTB)
  E *P = T + nb * nb;
  const long long b = blockIdx.x;
  const E *Gb = G + b * (long long)nb * nb;
  const E *tb = tau + b * sTau;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5, nw = blockDim.x >> 5;
  for (int q = tid; q < nb * nb; q += blockDim.x) T[q] = X::zero();
  __syncthreads();
  const int nblk = (nb + kTB - 1) / kTB;
  // 1. diagonal blocks: lane j < kTB owns row j0 + j of block d
  for (int d = wid; d < nblk; d += nw) {
    const int j0 = d * kTB, bs = min(kTB, nb - j0);
    for (int ii = 0; ii < bs; ++ii) {
      const int i = j0 + ii;
      const E ti = i < nvalid ? tb[i] : X::zero();  // padded reflectors: tau = 0, H = I
      if (lane < ii) {
        E sum = X::zero();
        for (int l = j0 + lane; l < i; ++l) mac(sum, T[(j0 + lane) + l * nb], __ldg(Gb + l + i * nb));
        T[(j0 + lane) + i * nb] = X::neg(X::mul(ti, sum));
      }
      if (lane == 0) T[i + i * nb] = ti;
      __syncwarp();
    }
  }
  __syncthreads();
  // 2. block columns J = 1 .. nblk-1 (sequential): rows [0, c0), columns [c0, c0 + bs)
  for (int J = 1; J < nblk; ++J) {
    const int c0 = J * kTB, bs = min(kTB, nb - c0), r0 = c0;
    // P = G(0:r0, J) T(J, J)   (r0 x bs)
    for (int q = tid; q < r0 * bs; q += blockDim.x) {
      const int r = q % r0, c = q / r0;
      E sum = X::zero();
      for (int l = 0; l <= c; ++l) mac(sum, __ldg(Gb + r + (c0 + l) * nb), T[(c0 + l) + (c0 + c) * nb]);
      P[r + c * nb] = sum;
    }
    __syncthreads();
    // T(0:r0, J) = -T(0:r0, 0:r0) P   (T(0:r0, 0:r0) upper triangular)
    for (int q = tid; q < r0 * bs; q += blockDim.x) {
      const int r = q % r0, c = q / r0;
      E sum = X::zero();
      for (int l = r; l < r0; ++l) mac(sum, T[r + l * nb], P[l + c * nb]);
      T[r + (c0 + c) * nb] = X::neg(sum);
    }
    __syncthreads();
  }
  E *Thb = Th + b * (long long)nb * nb;
  for (int q = tid; q < nb * nb; q += blockDim.x) {
    const int r = q % nb, c = q / nb;  // Th(r, c) = conj(T(c, r)), or T itself (orgqr)
    Thb[q] = herm ? X::conj(T[c + r * nb]) : T[q];
  }
}

// C += D over the trailing block (C: ld ldc, batch stride sC; D: dense
// mp x nt, ld mp): the accumulate of the update C - V X, kept out of the
// GEMM epilogue (CUTLASS's transform epilogue reads a complex source 4x
// slower than the whole beta = 0 GEMM, profiles/r02/experiments)
template <class E>
__global__ void add_block_kernel(E *C, int ldc, long long sC, const E *D, int mp, int nt, long long L) {
  const long long per = (long long)mp * nt;
  for (long long idx = blockIdx.x * (long long)blockDim.x + threadIdx.x; idx < per * L;
       idx += (long long)gridDim.x * blockDim.x) {
    const long long b = idx / per;
    const int rem = (int)(idx - b * per);
    const int j = rem / mp, i = rem - j * mp;
    E &c = C[b * sC + (long long)j * ldc + i];
    const E d = D[idx];
    if constexpr (El<E>::kComplex) {
      c.x += d.x;
      c.y += d.y;
    } else {
      c += d;
    }
  }
}

// the first n columns of the m x m identity (xORGQR's starting point);
// padding rows lda > m untouched
template <class E>
__global__ void eye_kernel(E *A, long long sA, int lda, int m, int n, long long L) {
  using X = El<E>;
  const long long per = (long long)m * n;
  for (long long idx = blockIdx.x * (long long)blockDim.x + threadIdx.x; idx < per * L;
       idx += (long long)gridDim.x * blockDim.x) {
    const long long b = idx / per;
    const int rem = (int)(idx - b * per);
    const int c = rem / m, r = rem - c * m;
    A[b * sA + (long long)c * lda + r] = r == c ? X::one() : X::zero();
  }
}

}  // namespace wy

namespace host {

// widest tall single-SM class: fp32 256 x 64, complex 256 x 96
int wy_panel_width(bqr_dtype_t dt) { return dt == BQR_R32 ? 64 : 96; }

// per-matrix workspace (bytes) of one panel sweep with panel width nb
static size_t wy_bytes_per_matrix(bqr_dtype_t dt, int m, int n, int nb) {
  const size_t es = dt == BQR_R32 ? 4 : 8;
  const size_t V = (size_t)m * nb, G = (size_t)nb * nb, W = (size_t)nb * std::max(0, n - nb);
  // V X before the accumulate: complex data reuse the dead conj(V), G, T^H
  // and W (m <= 256: m_p n_t <= m_p nb + 2 nb^2 + nb n_t), real data need it
  const size_t D = dt == BQR_R32 ? (size_t)m * std::max(0, n - nb) : 0;
  return es * ((dt == BQR_R32 ? 1 : 2) * V + 2 * G + 2 * W + D) + 256;
}

// shapes the blocked variant can take: the TMA rows of V, C and W need
// 16-byte multiples (m, lda multiples of 4 fp32 / 2 complex); beyond one
// panel; at most the 256-row register-file panel classes
bool wy_supported(bqr_dtype_t dt, int m, int n, int lda) {
  const int q = dt == BQR_R32 ? 4 : 2;
  return (dt == BQR_R32 || dt == BQR_C64) && m >= n && m <= 256 && n > wy_panel_width(dt) && m % q == 0 &&
         lda % q == 0;
}

size_t wy_workspace_bytes(bqr_dtype_t dt, int m, int n, int chunk) {
  return chunk * wy_bytes_per_matrix(dt, m, n, wy_panel_width(dt)) + 1024;
}

template <class E>
static int add_block(E *C, int ldc, long long sC, const E *D, int mp, int nt, long long L, cudaStream_t stream) {
  const long long ne = (long long)L * mp * nt;
  wy::add_block_kernel<E><<<(unsigned)std::min<long long>((ne + 255) / 256, 148 * 64), 256, 0, stream>>>(
      C, ldc, sC, D, mp, nt, L);
  return cudaGetLastError() == cudaSuccess ? BQR_SUCCESS : BQR_ERR_CUDA;
}

template <class E>
static int geqrf_wy_t(int m, int n, long long batch, void *A, int lda, void *tau, void *work, size_t work_bytes,
                      cudaStream_t stream, const Plan *(*pick_panel)(int, int)) {
  using T = wy::Tr<E>;
  constexpr bool kC = El<E>::kComplex;
  const bqr_dtype_t dt = kC ? BQR_C64 : BQR_R32;
  const int nb = wy_panel_width(dt);
  const int kmax = std::min(m, n);
  const long long sA = (long long)lda * n;
  const size_t per = wy_bytes_per_matrix(dt, m, n, nb);
  long long chunk = (long long)(work_bytes / per);
  if (chunk < 1) return -9;
  chunk = std::min(chunk, batch);
  char *ws = reinterpret_cast<char *>((reinterpret_cast<uintptr_t>(work) + 255) & ~uintptr_t(255));
  using GRow = wy::Gemm<E, cutlass::layout::RowMajor>;
  using GCol = wy::Gemm<E, cutlass::layout::ColumnMajor>;
  for (long long b0 = 0; b0 < batch; b0 += chunk) {
    const long long L = std::min(chunk, batch - b0);
    E *Ab = reinterpret_cast<E *>(A) + b0 * sA;
    E *tb = reinterpret_cast<E *>(tau) + b0 * kmax;
    for (int k0 = 0; k0 < kmax; k0 += nb) {
      const int w = std::min(nb, kmax - k0), mp = m - k0, nt = n - k0 - w;
      const Plan *p = pick_panel(mp, w);
      if (!p) return BQR_ERR_NOT_SUPPORTED;
      Call c{Ab + k0 + (size_t)k0 * lda, tb + k0, L, mp, w, std::min(mp, w), lda, stream};
      c.strideA = sA;
      c.strideT = kmax;
      int st = p->geqrf(c);
      if (st != BQR_SUCCESS) return st;
      if (nt <= 0) continue;
      // workspace carve-up for this chunk (Vc = V for real data)
      E *V = reinterpret_cast<E *>(ws);
      E *Vc = kC ? V + (size_t)L * mp * w : V;
      E *G = Vc + (size_t)L * mp * w;
      E *Th = G + (size_t)L * w * w;
      E *W = Th + (size_t)L * w * w;
      E *X = W + (size_t)L * w * nt;
      E *Dw = kC ? Vc : X + (size_t)L * w * nt;  // Vc .. W are dead once X is formed
      const long long nv = (long long)L * mp * w;
      wy::extract_v_kernel<E><<<(unsigned)std::min<long long>((nv + 255) / 256, 148 * 64), 256, 0, stream>>>(
          Ab, sA, lda, k0, mp, w, L, V, Vc);
      if (cudaGetLastError() != cudaSuccess) return BQR_ERR_CUDA;
      const int64_t sV = (int64_t)mp * w, sG = (int64_t)w * w, sW = (int64_t)w * nt;
      // G = V^H V: A = conj(V)^T (row-major view of Vc), B = V
      st = GRow::run(w, w, mp, (int)L, Vc, mp, sV, V, mp, sV, G, w, sG, T::one(), T::zero(), stream);
      if (st != BQR_SUCCESS) return st;
      const size_t tsm = (size_t)(w * w + w * wy::kTB) * sizeof(E);  // T and P
      if (!ensure_smem(reinterpret_cast<const void *>(wy::larft_kernel<E>), tsm)) return BQR_ERR_CUDA;
      wy::larft_kernel<E><<<(unsigned)L, 256, tsm, stream>>>(G, tb + k0, kmax, w, Th);
      if (cudaGetLastError() != cudaSuccess) return BQR_ERR_CUDA;
      // W = V^H C, C = the trailing columns A[k0:m, k0+w:n]
      E *Cb = Ab + k0 + (size_t)(k0 + w) * lda;
      st = GRow::run(w, nt, mp, (int)L, Vc, mp, sV, Cb, lda, sA, W, w, sW, T::one(), T::zero(), stream);
      if (st != BQR_SUCCESS) return st;
      // X = T^H W
      st = GCol::run(w, nt, w, (int)L, Th, w, sG, W, w, sW, X, w, sW, T::one(), T::zero(), stream);
      if (st != BQR_SUCCESS) return st;
      // C = C - V X: D = -V X (beta = 0), then C += D
      const int64_t sD = (int64_t)mp * nt;
      st = GCol::run(mp, nt, w, (int)L, V, mp, sV, X, w, sW, Dw, mp, sD, T::mone(), T::zero(), stream);
      if (st != BQR_SUCCESS) return st;
      st = add_block(Cb, lda, sA, Dw, mp, nt, L, stream);
      if (st != BQR_SUCCESS) return st;
    }
  }
  return BQR_SUCCESS;
}

int geqrf_wy(bqr_dtype_t dt, int m, int n, long long batch, void *A, int lda, void *tau, void *work,
             size_t work_bytes, cudaStream_t stream, const Plan *(*pick_panel)(int, int)) {
  return dt == BQR_R32 ? geqrf_wy_t<float>(m, n, batch, A, lda, tau, work, work_bytes, stream, pick_panel)
                       : geqrf_wy_t<float2>(m, n, batch, A, lda, tau, work, work_bytes, stream, pick_panel);
}

// ---- xORGQR by panels (bqr_orgqr_batched beyond the single-SM classes):
// Q = Q_0 Q_1 ... Q_{p-1}, Q_j = I - V_j T_j V_j^H; starting from the first n
// columns of I, Q_j is applied backwards to rows / columns k0_j.. (the
// columns left of k0_j are still unit vectors that V_j^H maps to 0).
static size_t orgqr_wy_bytes_per_matrix(bqr_dtype_t dt, int m, int n, int k) {
  const size_t es = dt == BQR_R32 ? 4 : 8;
  const int nb = wy_panel_width(dt);
  size_t v = 0, t = 0;
  for (int k0 = 0; k0 < k; k0 += nb) {
    const int w = std::min(nb, (k - k0 + 3) & ~3);
    v += (size_t)(m - k0) * w;
    t += (size_t)w * w;
  }
  return es * ((dt == BQR_R32 ? 1 : 2) * v + t + (size_t)nb * nb + 2 * (size_t)nb * n + (size_t)m * n) + 256;
}

size_t orgqr_wy_workspace_bytes(bqr_dtype_t dt, int m, int n, int k, int chunk) {
  return chunk * orgqr_wy_bytes_per_matrix(dt, m, n, k) + 1024;
}

template <class E>
static int orgqr_wy_t(int m, int n, int k, long long batch, void *A, int lda, const void *tau, void *work,
                      size_t work_bytes, cudaStream_t stream) {
  using T = wy::Tr<E>;
  constexpr bool kC = El<E>::kComplex;
  const bqr_dtype_t dt = kC ? BQR_C64 : BQR_R32;
  const int nb = wy_panel_width(dt);
  const long long sA = (long long)lda * n;
  const size_t per = orgqr_wy_bytes_per_matrix(dt, m, n, k);
  long long chunk = (long long)(work_bytes / per);
  if (chunk < 1) return -10;
  chunk = std::min(chunk, batch);
  using GRow = wy::Gemm<E, cutlass::layout::RowMajor>;
  using GCol = wy::Gemm<E, cutlass::layout::ColumnMajor>;
  const int np = (k + nb - 1) / nb;
  // panel widths padded to the TMA's 16-byte row alignment with zero
  // reflectors (tau = 0, H = I): an odd last panel keeps the GEMM operands aligned
  const int al = kC ? 2 : 4;
  auto width = [&](int k0) { return std::min(nb, (k - k0 + al - 1) / al * al); };
  for (long long b0 = 0; b0 < batch; b0 += chunk) {
    const long long L = std::min(chunk, batch - b0);
    E *Ab = reinterpret_cast<E *>(A) + b0 * sA;
    const E *tb = reinterpret_cast<const E *>(tau) + b0 * n;
    E *ws = reinterpret_cast<E *>((reinterpret_cast<uintptr_t>(work) + 255) & ~uintptr_t(255));
    // carve: per panel V_j, Vc_j (L x (m - k0) x w) and T_j (L x w x w); G; W; X
    E *Vp[16], *Vcp[16], *Tp[16];
    if (np > 16) return BQR_ERR_NOT_SUPPORTED;
    E *cur = ws;
    for (int j = 0; j < np; ++j) {
      const int k0 = j * nb, w = width(k0), mj = m - k0;
      Vp[j] = cur;
      cur += (size_t)L * mj * w;
      Vcp[j] = kC ? cur : Vp[j];
      if (kC) cur += (size_t)L * mj * w;
      Tp[j] = cur;
      cur += (size_t)L * w * w;
    }
    E *G = cur;
    E *W = G + (size_t)L * nb * nb;
    E *X = W + (size_t)L * nb * n;
    E *Dw = X + (size_t)L * nb * n;
    // 1. V_j and T_j of every panel while A still holds the reflectors
    for (int j = 0; j < np; ++j) {
      const int k0 = j * nb, w = width(k0), mj = m - k0;
      const long long nv = (long long)L * mj * w;
      wy::extract_v_kernel<E><<<(unsigned)std::min<long long>((nv + 255) / 256, 148 * 64), 256, 0, stream>>>(
          Ab, sA, lda, k0, mj, w, L, Vp[j], Vcp[j], k - k0);
      if (cudaGetLastError() != cudaSuccess) return BQR_ERR_CUDA;
      const int64_t sV = (int64_t)mj * w, sG = (int64_t)w * w;
      int st = GRow::run(w, w, mj, (int)L, Vcp[j], mj, sV, Vp[j], mj, sV, G, w, sG, T::one(), T::zero(), stream);
      if (st != BQR_SUCCESS) return st;
      const size_t tsm = (size_t)(w * w + w * wy::kTB) * sizeof(E);
      if (!ensure_smem(reinterpret_cast<const void *>(wy::larft_kernel<E>), tsm)) return BQR_ERR_CUDA;
      wy::larft_kernel<E><<<(unsigned)L, 256, tsm, stream>>>(G, tb + k0, n, w, Tp[j], false, k - k0);
      if (cudaGetLastError() != cudaSuccess) return BQR_ERR_CUDA;
    }
    // 2. A <- I (m x n)
    const long long ne = (long long)L * m * n;
    wy::eye_kernel<E><<<(unsigned)std::min<long long>((ne + 255) / 256, 148 * 64), 256, 0, stream>>>(Ab, sA, lda, m,
                                                                                                       n, L);
    if (cudaGetLastError() != cudaSuccess) return BQR_ERR_CUDA;
    // 3. E[k0:m, k0:n] <- Q_j E[k0:m, k0:n], j = p-1 .. 0
    for (int j = np - 1; j >= 0; --j) {
      const int k0 = j * nb, w = width(k0), mj = m - k0, nc = n - k0;
      const int64_t sV = (int64_t)mj * w, sG = (int64_t)w * w, sW = (int64_t)w * nc;
      E *Eb = Ab + k0 + (size_t)k0 * lda;
      int st = GRow::run(w, nc, mj, (int)L, Vcp[j], mj, sV, Eb, lda, sA, W, w, sW, T::one(), T::zero(), stream);
      if (st != BQR_SUCCESS) return st;
      st = GCol::run(w, nc, w, (int)L, Tp[j], w, sG, W, w, sW, X, w, sW, T::one(), T::zero(), stream);
      if (st != BQR_SUCCESS) return st;
      st = GCol::run(mj, nc, w, (int)L, Vp[j], mj, sV, X, w, sW, Dw, mj, (int64_t)mj * nc, T::mone(), T::zero(),
                     stream);
      if (st != BQR_SUCCESS) return st;
      st = add_block(Eb, lda, sA, Dw, mj, nc, L, stream);
      if (st != BQR_SUCCESS) return st;
    }
  }
  return BQR_SUCCESS;
}

int orgqr_wy(bqr_dtype_t dt, int m, int n, int k, long long batch, void *A, int lda, const void *tau, void *work,
             size_t work_bytes, cudaStream_t stream) {
  return dt == BQR_R32 ? orgqr_wy_t<float>(m, n, k, batch, A, lda, tau, work, work_bytes, stream)
                       : orgqr_wy_t<float2>(m, n, k, batch, A, lda, tau, work, work_bytes, stream);
}

}  // namespace host
}  // namespace bqr
#endif  // BQR_NO_CUTLASS

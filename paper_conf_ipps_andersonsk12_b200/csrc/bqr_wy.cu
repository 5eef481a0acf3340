// bqr_wy.cu -- compact-WY blocked QR for complex matrices beyond one SM
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
// The workspace is caller-owned device memory (bqr_geqrf_wy_batched); the
// batch is processed in chunks that fit it.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>

#include "bqr_launch.cuh"

#ifdef BQR_NO_CUTLASS
namespace bqr {
namespace host {
bool wy_supported(bqr_dtype_t, int, int, int) { return false; }
size_t wy_workspace_bytes(int, int, int, int) { return 0; }
int geqrf_wy(int, int, long long, void *, int, void *, void *, size_t, int, cudaStream_t,
             const Plan *(*)(int, int)) {
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

using Cf = cutlass::complex<float>;

// batched complex GEMM D = alpha A B + beta C on tcgen05 (FastF32 emulation)
template <class LayoutA>
struct Gemm {
  using LayoutB = cutlass::layout::ColumnMajor;
  using LayoutC = cutlass::layout::ColumnMajor;
  using MmaTileShape = cute::Shape<cute::_128, cute::_64, cute::_16>;
  using ClusterShape = cute::Shape<cute::_1, cute::_1, cute::_1>;
  using Epi = typename cutlass::epilogue::collective::CollectiveBuilder<
      cutlass::arch::Sm100, cutlass::arch::OpClassTensorOp, MmaTileShape, ClusterShape,
      cutlass::epilogue::collective::EpilogueTileAuto, Cf, Cf, Cf, LayoutC, 2, Cf, LayoutC, 2,
      cutlass::epilogue::FastF32NoSmemWarpSpecialized1Sm>::CollectiveOp;
  using Main = typename cutlass::gemm::collective::CollectiveBuilder<
      cutlass::arch::Sm100, cutlass::arch::OpClassTensorOp, Cf, LayoutA, 2, Cf, LayoutB, 2, Cf, MmaTileShape,
      ClusterShape,
      cutlass::gemm::collective::StageCountAutoCarveout<static_cast<int>(sizeof(typename Epi::SharedStorage))>,
      cutlass::gemm::KernelTmaWarpSpecialized1SmFastFP32Sm100>::CollectiveOp;
  using Kernel = cutlass::gemm::kernel::GemmUniversal<cute::Shape<int, int, int, int>, Main, Epi>;
  using Op = cutlass::gemm::device::GemmUniversalAdapter<Kernel>;

  // A: M x K (row-major: element (i, k) at i*lda + k; column-major: i + k*lda),
  // B: K x N column-major, C/D: M x N column-major; per-matrix strides s*.
  static int run(int M, int N, int K, int L, const Cf *A, int64_t lda, int64_t sA, const Cf *B, int64_t ldb,
                 int64_t sB, Cf *C, int64_t ldc, int64_t sC, Cf alpha, Cf beta, cudaStream_t stream) {
    typename Kernel::StrideA stA;
    if constexpr (cute::is_same_v<LayoutA, cutlass::layout::RowMajor>)
      stA = cute::make_stride(lda, cute::Int<1>{}, sA);
    else
      stA = cute::make_stride(cute::Int<1>{}, lda, sA);
    const typename Kernel::StrideB stB = cute::make_stride(ldb, cute::Int<1>{}, sB);
    const typename Kernel::StrideC stC = cute::make_stride(cute::Int<1>{}, ldc, sC);
    typename Op::Arguments args{cutlass::gemm::GemmUniversalMode::kGemm,
                                {M, N, K, L},
                                {A, stA, B, stB},
                                {{alpha, beta}, C, stC, C, stC}};
    Op op;
    if (Op::get_workspace_size(args) != 0) return BQR_ERR_NOT_SUPPORTED;  // data-parallel tiles need none
    if (op.can_implement(args) != cutlass::Status::kSuccess) return BQR_ERR_NOT_SUPPORTED;
    if (op.initialize(args, nullptr, stream) != cutlass::Status::kSuccess) return BQR_ERR_CUDA;
    if (op.run(stream) != cutlass::Status::kSuccess) return BQR_ERR_CUDA;
    return cudaGetLastError() == cudaSuccess ? BQR_SUCCESS : BQR_ERR_CUDA;
  }
};
using GemmRowA = Gemm<cutlass::layout::RowMajor>;
using GemmColA = Gemm<cutlass::layout::ColumnMajor>;

// V (m_p x nb, unit lower trapezoidal) and conj(V) of each matrix's panel
__global__ void extract_v_kernel(const float2 *A, long long sA, int lda, int k0, int mp, int nb, long long L,
                                 float2 *V, float2 *Vc) {
  const long long per = (long long)mp * nb;
  for (long long idx = blockIdx.x * (long long)blockDim.x + threadIdx.x; idx < per * L;
       idx += (long long)gridDim.x * blockDim.x) {
    const long long b = idx / per;
    const int rem = (int)(idx - b * per);
    const int i = rem / mp, r = rem - i * mp;  // column i, row r
    float2 v = make_float2(r == i ? 1.f : 0.f, 0.f);
    if (r > i) v = A[b * sA + (long long)(k0 + i) * lda + (k0 + r)];
    V[idx] = v;
    Vc[idx] = make_float2(v.x, -v.y);
  }
}

// xLARFT (forward, columnwise): T upper triangular with H_0 ... H_{nb-1} =
// I - V T V^H, from G = V^H V and tau, blocked for parallelism: the 16 x 16
// diagonal blocks by the column recurrence T(i, i) = tau_i,
// T(j, i) = -tau_i sum_{j <= l < i} T(j, l) G(l, i) (one warp each), then
// block column by block column T(0:J, J) = -T(0:J, 0:J) G(0:J, J) T(J, J)
// (the product of two compact-WY factors [V1 V2]: T12 = -T11 V1^H V2 T22).
// Writes Th = T^H (nb x nb, column-major).  One CTA per matrix.
constexpr int kTB = 16;
__global__ void __launch_bounds__(256) larft_kernel(const float2 *G, const float2 *tau, long long sTau, int nb,
                                                    float2 *Th) {
  extern __shared__ float2 T[];  // nb x nb column-major, then P (nb x kTB)
  float2 *P = T + nb * nb;
  const long long b = blockIdx.x;
  const float2 *Gb = G + b * (long long)nb * nb;
  const float2 *tb = tau + b * sTau;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5, nw = blockDim.x >> 5;
  for (int q = tid; q < nb * nb; q += blockDim.x) T[q] = make_float2(0.f, 0.f);
  __syncthreads();
  const int nblk = (nb + kTB - 1) / kTB;
  // 1. diagonal blocks: lane j < kTB owns row j0 + j of block d
  for (int d = wid; d < nblk; d += nw) {
    const int j0 = d * kTB, bs = min(kTB, nb - j0);
    for (int ii = 0; ii < bs; ++ii) {
      const int i = j0 + ii;
      const float2 ti = tb[i];
      float sr = 0.f, si = 0.f;
      if (lane < ii) {
        for (int l = j0 + lane; l < i; ++l) {
          const float2 a = T[(j0 + lane) + l * nb], g = __ldg(Gb + l + i * nb);
          sr = fmaf(a.x, g.x, fmaf(-a.y, g.y, sr));
          si = fmaf(a.x, g.y, fmaf(a.y, g.x, si));
        }
        // -tau_i * (sum)
        T[(j0 + lane) + i * nb] = make_float2(-(ti.x * sr - ti.y * si), -(ti.x * si + ti.y * sr));
      }
      if (lane == 0) T[i + i * nb] = ti;
      __syncwarp();
    }
  }
  __syncthreads();
  // 2. block columns J = 1 .. nblk-1 (sequential): rows [0, r0), columns [c0, c0 + bs)
  for (int J = 1; J < nblk; ++J) {
    const int c0 = J * kTB, bs = min(kTB, nb - c0), r0 = c0;
    // P = G(0:r0, J) T(J, J)   (r0 x bs)
    for (int q = tid; q < r0 * bs; q += blockDim.x) {
      const int r = q % r0, c = q / r0;
      float sr = 0.f, si = 0.f;
      for (int l = 0; l <= c; ++l) {  // T(J, J) upper triangular
        const float2 g = __ldg(Gb + r + (c0 + l) * nb), t = T[(c0 + l) + (c0 + c) * nb];
        sr = fmaf(g.x, t.x, fmaf(-g.y, t.y, sr));
        si = fmaf(g.x, t.y, fmaf(g.y, t.x, si));
      }
      P[r + c * nb] = make_float2(sr, si);
    }
    __syncthreads();
    // T(0:r0, J) = -T(0:r0, 0:r0) P   (T(0:r0, 0:r0) upper triangular)
    for (int q = tid; q < r0 * bs; q += blockDim.x) {
      const int r = q % r0, c = q / r0;
      float sr = 0.f, si = 0.f;
      for (int l = r; l < r0; ++l) {
        const float2 a = T[r + l * nb], p = P[l + c * nb];
        sr = fmaf(a.x, p.x, fmaf(-a.y, p.y, sr));
        si = fmaf(a.x, p.y, fmaf(a.y, p.x, si));
      }
      T[r + (c0 + c) * nb] = make_float2(-sr, -si);
    }
    __syncthreads();
  }
  float2 *Thb = Th + b * (long long)nb * nb;
  for (int q = tid; q < nb * nb; q += blockDim.x) {
    const int r = q % nb, c = q / nb;  // Th(r, c) = conj(T(c, r))
    const float2 v = T[c + r * nb];
    Thb[q] = make_float2(v.x, -v.y);
  }
}

}  // namespace wy

namespace host {

// per-matrix workspace (bytes) of one panel sweep with panel width nb
static size_t wy_bytes_per_matrix(int m, int n, int nb) {
  const size_t V = (size_t)m * nb, G = (size_t)nb * nb, W = (size_t)nb * std::max(0, n - nb);
  return 8 * (2 * V + 2 * G + 2 * W);
}

bool wy_supported(bqr_dtype_t dt, int m, int n, int lda) {
  return dt == BQR_C64 && m >= n && m <= 256 && n > 160 && m % 2 == 0 && lda % 2 == 0;
}

size_t wy_workspace_bytes(int m, int n, int chunk, int nb) { return chunk * wy_bytes_per_matrix(m, n, nb) + 1024; }

int geqrf_wy(int m, int n, long long batch, void *A, int lda, void *tau, void *work, size_t work_bytes, int nb,
             cudaStream_t stream, const Plan *(*pick_panel)(int, int)) {
  using wy::Cf;
  const int kmax = std::min(m, n);
  const long long sA = (long long)lda * n;
  const size_t per = wy_bytes_per_matrix(m, n, nb);
  long long chunk = (long long)(work_bytes / per);
  if (chunk < 1) return -9;
  chunk = std::min(chunk, batch);
  char *ws = reinterpret_cast<char *>((reinterpret_cast<uintptr_t>(work) + 255) & ~uintptr_t(255));
  for (long long b0 = 0; b0 < batch; b0 += chunk) {
    const long long L = std::min(chunk, batch - b0);
    float2 *Ab = reinterpret_cast<float2 *>(A) + b0 * sA;
    float2 *tb = reinterpret_cast<float2 *>(tau) + b0 * kmax;
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
      // workspace carve-up for this chunk
      float2 *V = reinterpret_cast<float2 *>(ws);
      float2 *Vc = V + (size_t)L * mp * w;
      float2 *G = Vc + (size_t)L * mp * w;
      float2 *Th = G + (size_t)L * w * w;
      float2 *W = Th + (size_t)L * w * w;
      float2 *X = W + (size_t)L * w * nt;
      const long long nv = (long long)L * mp * w;
      wy::extract_v_kernel<<<(unsigned)std::min<long long>((nv + 255) / 256, 148 * 64), 256, 0, stream>>>(
          Ab, sA, lda, k0, mp, w, L, V, Vc);
      if (cudaGetLastError() != cudaSuccess) return BQR_ERR_CUDA;
      const Cf one(1.f, 0.f), zero(0.f, 0.f), mone(-1.f, 0.f);
      const int64_t sV = (int64_t)mp * w, sG = (int64_t)w * w, sW = (int64_t)w * nt;
      // G = V^H V: A = conj(V)^T (row-major view of Vc), B = V
      st = wy::GemmRowA::run(w, w, mp, (int)L, reinterpret_cast<Cf *>(Vc), mp, sV, reinterpret_cast<Cf *>(V), mp, sV,
                             reinterpret_cast<Cf *>(G), w, sG, one, zero, stream);
      if (st != BQR_SUCCESS) return st;
      const size_t tsm = (size_t)(w * w + w * wy::kTB) * sizeof(float2);  // T and P: > 48 KB for nb = 96
      if (!ensure_smem(reinterpret_cast<const void *>(wy::larft_kernel), tsm)) return BQR_ERR_CUDA;
      wy::larft_kernel<<<(unsigned)L, 256, tsm, stream>>>(G, tb + k0, kmax, w, Th);
      if (cudaGetLastError() != cudaSuccess) return BQR_ERR_CUDA;
      // W = V^H C, C = the trailing columns A[k0:m, k0+w:n]
      Cf *Cb = reinterpret_cast<Cf *>(Ab + k0 + (size_t)(k0 + w) * lda);
      st = wy::GemmRowA::run(w, nt, mp, (int)L, reinterpret_cast<Cf *>(Vc), mp, sV, Cb, lda, sA,
                             reinterpret_cast<Cf *>(W), w, sW, one, zero, stream);
      if (st != BQR_SUCCESS) return st;
      // X = T^H W
      st = wy::GemmColA::run(w, nt, w, (int)L, reinterpret_cast<Cf *>(Th), w, sG, reinterpret_cast<Cf *>(W), w, sW,
                             reinterpret_cast<Cf *>(X), w, sW, one, zero, stream);
      if (st != BQR_SUCCESS) return st;
      // C = C - V X
      st = wy::GemmColA::run(mp, nt, w, (int)L, reinterpret_cast<Cf *>(V), mp, sV, reinterpret_cast<Cf *>(X), w, sW,
                             Cb, lda, sA, mone, one, stream);
      if (st != BQR_SUCCESS) return st;
    }
  }
  return BQR_SUCCESS;
}

}  // namespace host
}  // namespace bqr
#endif  // BQR_NO_CUTLASS

// Probe: batched complex-fp32 GEMM on tcgen05 tensor cores through CUTLASS's
// SM100 FastF32 (BF16-split emulation of FP32) collective, the candidate
// engine for the compact-WY trailing update C <- C - V (T^H (V^H C)) of the
// blocked QR variant (north-star).  Checks accuracy against a
// CUDA-core fp32 reference on the shapes the WY update produces and times it.
//   nvcc -std=c++17 -O3 -gencode arch=compute_100a,code=sm_100a -I<cutlass>/include
//        -I<cutlass>/tools/util/include --expt-relaxed-constexpr tools/micro/wy_gemm_probe.cu -lcuda
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cmath>

#include "cutlass/cutlass.h"
#include "cute/tensor.hpp"
#include "cutlass/complex.h"
#include "cutlass/gemm/dispatch_policy.hpp"
#include "cutlass/gemm/collective/collective_builder.hpp"
#include "cutlass/epilogue/collective/collective_builder.hpp"
#include "cutlass/gemm/kernel/gemm_universal.hpp"
#include "cutlass/gemm/device/gemm_universal_adapter.h"

using namespace cute;
using Cf = cutlass::complex<float>;

template <class LayoutA, class LayoutB, bool TWO_SM = false>
struct FastGemm {
  using LayoutC = cutlass::layout::ColumnMajor;
  using MmaTileShape = cute::conditional_t<TWO_SM, Shape<_256, _64, _16>, Shape<_128, _64, _16>>;
  using ClusterShape = cute::conditional_t<TWO_SM, Shape<_2, _1, _1>, Shape<_1, _1, _1>>;
  using EpiSched = cute::conditional_t<TWO_SM, cutlass::epilogue::FastF32NoSmemWarpSpecialized2Sm,
                                       cutlass::epilogue::FastF32NoSmemWarpSpecialized1Sm>;
  using MainSched = cute::conditional_t<TWO_SM, cutlass::gemm::KernelTmaWarpSpecialized2SmFastFP32Sm100,
                                        cutlass::gemm::KernelTmaWarpSpecialized1SmFastFP32Sm100>;
  using CollectiveEpilogue = typename cutlass::epilogue::collective::CollectiveBuilder<
      cutlass::arch::Sm100, cutlass::arch::OpClassTensorOp, MmaTileShape, ClusterShape,
      cutlass::epilogue::collective::EpilogueTileAuto, Cf, Cf, Cf, LayoutC, 2, Cf, LayoutC, 2,
      EpiSched>::CollectiveOp;
  using CollectiveMainloop = typename cutlass::gemm::collective::CollectiveBuilder<
      cutlass::arch::Sm100, cutlass::arch::OpClassTensorOp, Cf, LayoutA, 2, Cf, LayoutB, 2, Cf, MmaTileShape,
      ClusterShape,
      cutlass::gemm::collective::StageCountAutoCarveout<static_cast<int>(
          sizeof(typename CollectiveEpilogue::SharedStorage))>,
      MainSched>::CollectiveOp;
  using Kernel = cutlass::gemm::kernel::GemmUniversal<Shape<int, int, int, int>, CollectiveMainloop,
                                                      CollectiveEpilogue>;
  using Gemm = cutlass::gemm::device::GemmUniversalAdapter<Kernel>;
  using StrideA = typename Kernel::StrideA;
  using StrideB = typename Kernel::StrideB;
  using StrideC = typename Kernel::StrideC;
  using StrideD = typename Kernel::StrideD;
};

// reference: D = alpha op(A) B + beta C, A row-major (M x K, lda, = K-major) if TA else column-major
__global__ void ref_gemm(int M, int N, int K, int L, const Cf *A, long long lda, long long sA, bool a_rowmajor,
                         const Cf *B, long long ldb, long long sB, const Cf *C, long long ldc, long long sC, Cf *D,
                         Cf alpha, Cf beta) {
  long long idx = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  long long tot = (long long)M * N * L;
  if (idx >= tot) return;
  int i = idx % M, j = (idx / M) % N, l = idx / ((long long)M * N);
  double ar = 0, ai = 0;
  for (int k = 0; k < K; ++k) {
    Cf a = a_rowmajor ? A[l * sA + (long long)i * lda + k] : A[l * sA + i + (long long)k * lda];
    Cf b = B[l * sB + k + (long long)j * ldb];
    ar += (double)a.real() * b.real() - (double)a.imag() * b.imag();
    ai += (double)a.real() * b.imag() + (double)a.imag() * b.real();
  }
  Cf c = C[l * sC + i + (long long)j * ldc];
  double dr = alpha.real() * ar - alpha.imag() * ai + beta.real() * c.real() - beta.imag() * c.imag();
  double di = alpha.real() * ai + alpha.imag() * ar + beta.real() * c.imag() + beta.imag() * c.real();
  D[l * sC + i + (long long)j * ldc] = Cf((float)dr, (float)di);
}

template <class G>
int run(const char *name, int M, int N, int K, int L, bool a_rowmajor) {
  using Gemm = typename G::Gemm;
  const int64_t lda = a_rowmajor ? K : M, ldb = K, ldc = M;
  const int64_t sA = (int64_t)M * K, sB = (int64_t)K * N, sC = (int64_t)M * N;
  std::vector<Cf> hA(sA * L), hB(sB * L), hC(sC * L);
  srand(1);
  auto rnd = [] { return (float)rand() / RAND_MAX - 0.5f; };
  for (auto &x : hA) x = Cf(rnd(), rnd());
  for (auto &x : hB) x = Cf(rnd(), rnd());
  for (auto &x : hC) x = Cf(rnd(), rnd());
  Cf *dA, *dB, *dC, *dD, *dR;
  cudaMalloc(&dA, hA.size() * 8);
  cudaMalloc(&dB, hB.size() * 8);
  cudaMalloc(&dC, hC.size() * 8);
  cudaMalloc(&dD, hC.size() * 8);
  cudaMalloc(&dR, hC.size() * 8);
  cudaMemcpy(dA, hA.data(), hA.size() * 8, cudaMemcpyHostToDevice);
  cudaMemcpy(dB, hB.data(), hB.size() * 8, cudaMemcpyHostToDevice);
  cudaMemcpy(dC, hC.data(), hC.size() * 8, cudaMemcpyHostToDevice);
  Cf alpha(-1.f, 0.f), beta(1.f, 0.f);
  typename G::StrideA strideA;
  typename G::StrideB strideB;
  typename G::StrideC strideC;
  typename G::StrideD strideD;
  // fill the dynamic strides (static unit strides are implicit)
  if constexpr (cute::is_same_v<typename G::StrideA, cute::Stride<int64_t, cute::Int<1>, int64_t>>)
    strideA = cute::make_stride(lda, cute::Int<1>{}, sA);
  else
    strideA = cute::make_stride(cute::Int<1>{}, lda, sA);
  strideB = cute::make_stride(ldb, cute::Int<1>{}, sB);
  strideC = cute::make_stride(cute::Int<1>{}, ldc, sC);
  strideD = strideC;
  typename Gemm::Arguments args{cutlass::gemm::GemmUniversalMode::kGemm,
                                {M, N, K, L},
                                {dA, strideA, dB, strideB},
                                {{alpha, beta}, dC, strideC, dD, strideD}};
  Gemm gemm;
  size_t ws = Gemm::get_workspace_size(args);
  void *dws = nullptr;
  if (ws) cudaMalloc(&dws, ws);
  cutlass::Status st = gemm.can_implement(args);
  if (st != cutlass::Status::kSuccess) {
    printf("{\"probe\":\"%s\",\"error\":\"can_implement %d\"}\n", name, (int)st);
    return 1;
  }
  st = gemm.initialize(args, dws);
  if (st != cutlass::Status::kSuccess) {
    printf("{\"probe\":\"%s\",\"error\":\"initialize %d\"}\n", name, (int)st);
    return 1;
  }
  st = gemm.run();
  cudaError_t e = cudaDeviceSynchronize();
  if (st != cutlass::Status::kSuccess || e != cudaSuccess) {
    printf("{\"probe\":\"%s\",\"error\":\"run %d %s\"}\n", name, (int)st, cudaGetErrorString(e));
    return 1;
  }
  long long tot = sC * L;
  ref_gemm<<<(tot + 255) / 256, 256>>>(M, N, K, L, dA, lda, sA, a_rowmajor, dB, ldb, sB, dC, ldc, sC, dR, alpha, beta);
  cudaDeviceSynchronize();
  std::vector<Cf> hD(tot), hR(tot);
  cudaMemcpy(hD.data(), dD, tot * 8, cudaMemcpyDeviceToHost);
  cudaMemcpy(hR.data(), dR, tot * 8, cudaMemcpyDeviceToHost);
  double maxerr = 0, maxref = 0;
  for (long long i = 0; i < tot; ++i) {
    maxerr = fmax(maxerr, cutlass::abs(hD[i] - hR[i]));
    maxref = fmax(maxref, cutlass::abs(hR[i]));
  }
  // timing
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int i = 0; i < 3; ++i) gemm.run();
  cudaEventRecord(e0);
  const int reps = 20;
  for (int i = 0; i < reps; ++i) gemm.run();
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  ms /= reps;
  double flops = 8.0 * M * N * K * L;
  printf("{\"probe\":\"%s\",\"M\":%d,\"N\":%d,\"K\":%d,\"L\":%d,\"max_abs_err\":%.3e,\"max_ref\":%.3e,\"rel\":%.3e,"
         "\"us\":%.2f,\"tflops\":%.2f}\n",
         name, M, N, K, L, maxerr, maxref, maxerr / maxref / sqrt((double)K), ms * 1e3, flops / ms / 1e9);
  cudaFree(dA);
  cudaFree(dB);
  cudaFree(dC);
  cudaFree(dD);
  cudaFree(dR);
  if (dws) cudaFree(dws);
  return 0;
}

int main() {
  using GRow = FastGemm<cutlass::layout::RowMajor, cutlass::layout::ColumnMajor>;   // W = Vc^T B (A K-major)
  using GCol = FastGemm<cutlass::layout::ColumnMajor, cutlass::layout::ColumnMajor>; // C -= V W' (A M-major)
  using GCol2 = FastGemm<cutlass::layout::ColumnMajor, cutlass::layout::ColumnMajor, true>;
  run<GRow>("W=VhC_256x96x160", 96, 160, 256, 2368, true);
  run<GCol>("C-=VW_256x160x96", 256, 160, 96, 2368, false);
  run<GCol2>("C-=VW_256x160x96_2sm", 256, 160, 96, 2368, false);
  run<GRow>("W=VhC_192x96x96", 96, 96, 192, 2368, true);
  run<GCol>("C-=VW_192x96x96", 192, 96, 96, 2368, false);
  return 0;
}

// bqr_solve.cu -- the triangular solve of the least-squares path
// (bqr_gels_batched): X = R^{-1} (Q^H B)[0:n] by backward elimination.
//
// Paper Sec. III-D: "Rx = Q^T b ... We compute Q^T b by
// appending b to the right side of the matrix during the factorization.  We
// then solve the upper triangular system using row operations."  The row
// operations are column-oriented back substitution on [R | c]: for
// j = n-1 .. 0, x_j = c_j / R_jj (IEEE division), then c_i -= R_ij x_j for
// every row i < j (row j times x_j subtracted from the rows above).
//
// B200 mapping: one warp per matrix (grid-stride over the batch).  The upper
// triangle of R is staged once into shared memory, packed by column (column
// j's rows 0..j at offset j(j+1)/2, so each step reads a contiguous,
// conflict-free column); c is held cyclically over the 32 lanes (element i
// in lane i % 32, register i / 32).  Per step: one shuffle broadcasts c_j,
// every lane divides by the (broadcast) diagonal, the owner lane stores x_j,
// and each lane updates its rows i < j with one FMA per row.  The n-step
// dependent chain (shuffle + IEEE division) is the latency floor; the batch
// supplies the parallelism.  Matrices whose packed triangle exceeds the
// shared-memory budget (complex n > 226) read R from global memory instead.
#include "bqr_launch.cuh"

namespace bqr {

struct SolveArgs {
  const void *A;  // R in the upper triangle (geqrf output)
  void *B;        // in: (Q^H B); out: rows 0..n-1 = X
  int *info;      // per matrix: 0, or j+1 for the first R_jj == 0 (may be null)
  long long batch;
  int n, lda, ldb, nrhs;
  long long strideA, strideB;
};

template <class T, int NT, bool STAGED>
__global__ void __launch_bounds__(32) solve_upper_kernel(const SolveArgs p) {
  using X = El<T>;
  extern __shared__ __align__(16) float smem_f[];
  T *sR = reinterpret_cast<T *>(smem_f);
  const int lane = threadIdx.x;
  const int n = p.n;
  for (long long b = blockIdx.x; b < p.batch; b += gridDim.x) {
    const T *R = reinterpret_cast<const T *>(p.A) + b * p.strideA;
    if constexpr (STAGED) {
      __syncwarp();  // previous matrix fully consumed
      for (int j = 0; j < n; ++j) {
        const int base = j * (j + 1) / 2;
        for (int i = lane; i <= j; i += 32) sR[base + i] = R[i + (long long)j * p.lda];
      }
      __syncwarp();
    }
    auto rget = [&](int i, int j) -> T {
      if constexpr (STAGED) {
        return sR[j * (j + 1) / 2 + i];
      } else {
        return R[i + (long long)j * p.lda];
      }
    };
    // first zero diagonal (LAPACK xTRTRS info): lanes scan i = lane + 32 t
    int first = 0x7fffffff;
#pragma unroll
    for (int t = 0; t < NT; ++t) {
      const int i = lane + 32 * t;
      if (i < n) {
        const T d = rget(i, i);
        if (X::re(d) == 0.f && X::im(d) == 0.f && i < first) first = i;
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) first = min(first, __shfl_xor_sync(0xffffffffu, first, o));
    if (p.info && lane == 0) p.info[b] = first == 0x7fffffff ? 0 : first + 1;

    for (int r = 0; r < p.nrhs; ++r) {
      T *c = reinterpret_cast<T *>(p.B) + b * p.strideB + (long long)r * p.ldb;
      T x[NT];
#pragma unroll
      for (int t = 0; t < NT; ++t) {
        const int i = lane + 32 * t;
        x[t] = i < n ? c[i] : X::zero();
      }
#pragma unroll 1
      for (int j = n - 1; j >= 0; --j) {
        const int tj = j >> 5, oj = j & 31;
        T cj = x[0];
#pragma unroll
        for (int t = 1; t < NT; ++t) cj = X::sel(t == tj, x[t], cj);
        cj = X::shfl(cj, oj);
        // the diagonal of a geqrf R is real (LAPACK; imag exactly 0):
        // IEEE division of each component by it
        const float d = X::re(rget(j, j));
        const T xj = X::make(X::re(cj) / d, X::im(cj) / d);
#pragma unroll
        for (int t = 0; t < NT; ++t) {
          const int i = lane + 32 * t;
          if (t == tj && lane == oj) x[t] = xj;
          if (i < j) x[t] = X::fnms(rget(i, j), xj, x[t]);
        }
      }
#pragma unroll
      for (int t = 0; t < NT; ++t) {
        const int i = lane + 32 * t;
        if (i < n) c[i] = x[t];
      }
    }
  }
}

namespace host {

template <class T, int NT>
int launch_solve(const SolveArgs &a, cudaStream_t s) {
  const size_t packed = (size_t)a.n * (a.n + 1) / 2 * sizeof(T);
  const bool staged = packed <= 200 * 1024;
  const void *kern = staged ? reinterpret_cast<const void *>(solve_upper_kernel<T, NT, true>)
                            : reinterpret_cast<const void *>(solve_upper_kernel<T, NT, false>);
  const size_t smem = staged ? packed : 0;
  if (!ensure_smem(kern, smem)) return BQR_ERR_CUDA;
  int sms = 0, bps = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, current_device());
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, kern, 32, smem);
  const long long grid = std::min<long long>(a.batch, (long long)std::max(1, sms) * std::max(1, bps));
  if (staged) {
    solve_upper_kernel<T, NT, true><<<(unsigned)grid, 32, smem, s>>>(a);
  } else {
    solve_upper_kernel<T, NT, false><<<(unsigned)grid, 32, 0, s>>>(a);
  }
  return finish_launch();
}

template <class T>
int solve_dispatch_t(const SolveArgs &a, cudaStream_t s) {
  if (a.n <= 32) return launch_solve<T, 1>(a, s);
  if (a.n <= 64) return launch_solve<T, 2>(a, s);
  if (a.n <= 128) return launch_solve<T, 4>(a, s);
  if (a.n <= 256) return launch_solve<T, 8>(a, s);
  return BQR_ERR_NOT_SUPPORTED;
}

int solve_upper_dispatch(bqr_dtype_t dt, const void *A, int lda, long long strideA, void *B, int ldb,
                         long long strideB, int *info, long long batch, int n, int nrhs, cudaStream_t s) {
  SolveArgs a{A, B, info, batch, n, lda, ldb, nrhs, strideA, strideB};
  return dt == BQR_R32 ? solve_dispatch_t<float>(a, s) : solve_dispatch_t<float2>(a, s);
}

}  // namespace host
}  // namespace bqr

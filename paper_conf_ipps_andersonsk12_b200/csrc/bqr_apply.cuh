// bqr_apply.cuh -- B <- Q^H B from stored reflectors (xORM2R / xUNM2R,
// SIDE='L', TRANS='T'/'C').  The paper's least-squares step computes Q^T b
// by carrying b through the factorisation; as a separate call
// it is k reflector applications H_i^H = I - conj(tau_i) v_i v_i^H, in order
// i = 0 .. k-1.
//
// One warp per (matrix, block of NB right-hand sides): rows are cyclic over
// the 32 lanes (each warp access to a reflector column is a contiguous,
// coalesced segment), the NB dot products v^H B are warp-shuffle butterflies
// (no barrier), and the next reflector column is prefetched into registers
// while the current one is applied (V does not depend on B).
#pragma once
#include "bqr_common.cuh"

namespace bqr {

struct ApplyArgs {
  const void *A;
  const void *tau;
  void *B;
  long long batch;
  int lda, ncolsA, m, k, nrhs, ldb;
};

template <class T, int MR, int NB>
struct ApplyQh {
  using X = El<T>;
  static constexpr int kWarps = 4;

  static __device__ __forceinline__ void load_v(T (&v)[MR], const T *col, int i, int m, int lane) {
#pragma unroll
    for (int s = 0; s < MR; ++s) {
      const int r = lane + 32 * s;
      T x = X::zero();
      if (r > i && r < m) x = col[r];
      v[s] = X::sel(r == i, X::one(), x);
    }
  }

  static __device__ __forceinline__ void run(const ApplyArgs &p) {
    const int lane = threadIdx.x & 31;
    const int nblk = (p.nrhs + NB - 1) / NB;
    const long long item = (long long)blockIdx.x * kWarps + (threadIdx.x >> 5);
    if (item >= p.batch * nblk) return;
    const long long mat = item / nblk;
    const int j0 = (int)(item - mat * nblk) * NB;
    const T *Ab = reinterpret_cast<const T *>(p.A) + mat * (long long)p.lda * p.ncolsA;
    const T *tg = reinterpret_cast<const T *>(p.tau) + mat * (long long)p.k;
    T *Bb = reinterpret_cast<T *>(p.B) + mat * (long long)p.ldb * p.nrhs;
    T b[MR][NB];
#pragma unroll
    for (int s = 0; s < MR; ++s)
#pragma unroll
      for (int j = 0; j < NB; ++j) {
        const int r = lane + 32 * s;
        b[s][j] = (r < p.m && j0 + j < p.nrhs) ? Bb[r + (long long)(j0 + j) * p.ldb] : X::zero();
      }
    T v[MR], vn[MR];
    if (p.k > 0) load_v(v, Ab, 0, p.m, lane);
#pragma unroll 1
    for (int i = 0; i < p.k; ++i) {
      if (i + 1 < p.k) load_v(vn, Ab + (long long)(i + 1) * p.lda, i + 1, p.m, lane);
      const T ct = X::conj(tg[i]);
#pragma unroll
      for (int j = 0; j < NB; ++j) {
        T w = X::zero();
#pragma unroll
        for (int s = 0; s < MR; ++s) w = X::cfma(v[s], b[s][j], w);
        w = row_allreduce<32>(w);
        const T tw = X::mul(ct, w);
#pragma unroll
        for (int s = 0; s < MR; ++s) b[s][j] = X::fnms(v[s], tw, b[s][j]);
      }
#pragma unroll
      for (int s = 0; s < MR; ++s) v[s] = vn[s];
    }
#pragma unroll
    for (int s = 0; s < MR; ++s)
#pragma unroll
      for (int j = 0; j < NB; ++j) {
        const int r = lane + 32 * s;
        if (r < p.m && j0 + j < p.nrhs) Bb[r + (long long)(j0 + j) * p.ldb] = b[s][j];
      }
  }
};

template <class T, int MR, int NB>
__global__ void __launch_bounds__(128) apply_qh_kernel(const ApplyArgs p) {
  ApplyQh<T, MR, NB>::run(p);
}

}  // namespace bqr

// bqr_apply.cuh -- B <- Q^H B from stored reflectors (xORM2R / xUNM2R,
// SIDE='L', TRANS='T'/'C').  The paper's least-squares step computes Q^T b
// by carrying b through the factorisation; as a separate call
// it is k reflector applications H_i^H = I - conj(tau_i) v_i v_i^H, in order
// i = 0 .. k-1.
//
// One warp per (matrix, block of NB right-hand sides): rows are cyclic over
// the 32 lanes (each warp access to a reflector column is a contiguous,
// coalesced segment) and the NB dot products v^H B are warp-shuffle
// butterflies (no barrier).  V does not depend on B, so the reflector
// columns stream through a PF-deep register ring: column i+PF is requested
// while column i is applied, which hides the L2/HBM latency behind the
// serial chain of reflector applications.
#pragma once
#include "bqr_common.cuh"

namespace bqr {

struct ApplyArgs {
  const void *A;
  const void *tau;
  void *B;
  long long batch;
  int lda, ncolsA, m, k, nrhs, ldb;
  long long strideA, strideT, strideB;  // batch strides (elements)
};

template <class T, int MR, int NB, int PF>
struct ApplyQh {
  using X = El<T>;
  static constexpr int kWarps = MR >= 4 ? 1 : 4;  // long columns: one warp per CTA spreads the SMs

  // raw column (rows >= i); the v_i = 1 / zero-above masks are applied at
  // use time, so nothing consumes the load until the ring comes round
  // (asm volatile: ptxas otherwise sinks the loads to their first use, which
  // turns the prefetch ring back into one exposed memory latency per column)
  static __device__ __forceinline__ void ldg(float &d, const float *p, bool pred) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %2, 0;\n\t@q ld.global.nc.f32 %0, [%1];\n}"
                 : "+f"(d) : "l"(p), "r"((int)pred));
  }
  static __device__ __forceinline__ void ldg(float2 &d, const float2 *p, bool pred) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %3, 0;\n\t@q ld.global.nc.v2.f32 {%0, %1}, [%2];\n}"
                 : "+f"(d.x), "+f"(d.y) : "l"(p), "r"((int)pred));
  }
  static __device__ __forceinline__ void load_v(T (&v)[MR], const T *col, int i, int m, int lane) {
#pragma unroll
    for (int s = 0; s < MR; ++s) {
      const int r = lane + 32 * s;
      ldg(v[s], col + r, r >= i && r < m);
    }
  }

  static __device__ __forceinline__ void apply_one(T (&b)[MR][NB], const T (&raw)[MR], T ct, int i, int m, int lane) {
    T v[MR];
#pragma unroll
    for (int s = 0; s < MR; ++s) {
      const int r = lane + 32 * s;
      v[s] = X::sel(r > i && r < m, raw[s], X::sel(r == i, X::one(), X::zero()));
    }
#pragma unroll
    for (int j = 0; j < NB; ++j) {
      T w0 = X::zero(), w1 = X::zero();
#pragma unroll
      for (int s = 0; s < MR; ++s) {
        if (s & 1) w1 = X::cfma(v[s], b[s][j], w1);
        else w0 = X::cfma(v[s], b[s][j], w0);
      }
      const T w = row_allreduce<32>(X::add(w0, w1));
      const T tw = X::mul(ct, w);
#pragma unroll
      for (int s = 0; s < MR; ++s) b[s][j] = X::fnms(v[s], tw, b[s][j]);
    }
  }

  static __device__ __forceinline__ void run(const ApplyArgs &p) {
    const int lane = threadIdx.x & 31;
    const int nblk = (p.nrhs + NB - 1) / NB;
    const long long item = (long long)blockIdx.x * kWarps + (threadIdx.x >> 5);
    if (item >= p.batch * nblk) return;
    const long long mat = item / nblk;
    const int j0 = (int)(item - mat * nblk) * NB;
    const T *Ab = reinterpret_cast<const T *>(p.A) + mat * p.strideA;
    const T *tg = reinterpret_cast<const T *>(p.tau) + mat * p.strideT;
    T *Bb = reinterpret_cast<T *>(p.B) + mat * p.strideB;
    T b[MR][NB];
#pragma unroll
    for (int s = 0; s < MR; ++s)
#pragma unroll
      for (int j = 0; j < NB; ++j) {
        const int r = lane + 32 * s;
        b[s][j] = (r < p.m && j0 + j < p.nrhs) ? Bb[r + (long long)(j0 + j) * p.ldb] : X::zero();
      }
    T ring[PF][MR];
    T tr[PF];
#pragma unroll
    for (int q = 0; q < PF; ++q) {
#pragma unroll
      for (int s = 0; s < MR; ++s) ring[q][s] = X::zero();
      tr[q] = X::zero();
    }
#pragma unroll
    for (int q = 0; q < PF; ++q) {
      if (q < p.k) {
        load_v(ring[q], Ab + (long long)q * p.lda, q, p.m, lane);
        tr[q] = tg[q];
      }
    }
#pragma unroll 1
    for (int i0 = 0; i0 < p.k; i0 += PF) {
#pragma unroll
      for (int q = 0; q < PF; ++q) {
        const int i = i0 + q;
        if (i < p.k) {
          apply_one(b, ring[q], X::conj(tr[q]), i, p.m, lane);
          if (i + PF < p.k) {
            load_v(ring[q], Ab + (long long)(i + PF) * p.lda, i + PF, p.m, lane);
            ldg(tr[q], tg + i + PF, true);
          }
        }
      }
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

template <class T, int MR, int NB, int PF>
__global__ void __launch_bounds__(ApplyQh<T, MR, NB, PF>::kWarps * 32) apply_qh_kernel(const ApplyArgs p) {
  ApplyQh<T, MR, NB, PF>::run(p);
}

}  // namespace bqr

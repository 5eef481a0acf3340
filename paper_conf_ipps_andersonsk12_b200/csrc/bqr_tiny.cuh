// bqr_tiny.cuh -- one problem per thread for tiny matrices (m, n <= 8).
//
// The paper's Sec. IV: each thread holds its whole matrix in
// registers and factors it serially; performance is then "the product of the
// problem's arithmetic intensity and the global DRAM bandwidth",
// i.e. the path is HBM-bound and the only thing that matters is moving the
// batch at full bandwidth.  On GF100 the 64-register cap spilled n >= 8
// (P:L383); sm_100a allows 255 registers, so 8x8 fp32 (64 words) and 8x8 c64
// (128 words) stay in registers.
//
// B200 data movement: a warp owns 32 consecutive matrices, which are one
// contiguous 32*m*n*s-byte span when lda == m.  The warp reads that span with
// fully coalesced 16-byte loads, writes it to shared memory with an XOR
// swizzle on the 16-byte chunk index, then every thread reads its own
// matrix's chunks back conflict-free (chunk f = Q*lane + c lands in bank
// quad (f ^ (f / Q)) & 7, all distinct within a quarter warp), and the same in
// reverse for the store.  Other layouts (lda > m, misaligned base) take the
// per-thread direct path.
#pragma once
#include "bqr_common.cuh"

namespace bqr {

struct TinyArgs {
  void *A;
  void *tau;
  long long batch;
  int lda;
  int staged;  // lda == m, m*n*E % 4 == 0, 16-byte aligned base
};

template <class T, int M, int N>
struct Tiny {
  using X = El<T>;
  static constexpr int K = M < N ? M : N;
  static constexpr int E = sizeof(T) / 4;
  static constexpr int WORDS = M * N * E;        // 32-bit words per matrix
  static constexpr int Q = WORDS / 4;            // 16-byte chunks per matrix
  static constexpr bool kCanStage = (WORDS % 4 == 0) && Q >= 2;
  static constexpr int kWarps = WORDS <= 64 ? 4 : 2;  // warps per CTA (static smem <= 32 KB)
  static constexpr int kSmemWordsPerWarp = kCanStage ? 32 * WORDS : 1;

  static constexpr int QS = Q > 0 ? Q : 1;
  static __device__ __forceinline__ int swz(int f) { return (f & ~7) | ((f & 7) ^ ((f / QS) & 7)); }

  // serial xGEQR2 on a register-resident matrix (Table VI steps, one thread)
  static __device__ __forceinline__ void factor(T (&a)[M][N], T (&tau)[K]) {
#pragma unroll
    for (int k = 0; k < K; ++k) {
      float sig = 0.f;
#pragma unroll
      for (int r = k + 1; r < M; ++r) sig = X::abs2_acc(a[r][k], sig);
      const Reflector<T> h = make_reflector(a[k][k], sig);
#pragma unroll
      for (int r = k + 1; r < M; ++r) a[r][k] = X::mul(a[r][k], h.scal);
      a[k][k] = h.skip ? a[k][k] : X::make(h.beta, 0.f);
      tau[k] = h.tau;
      const T ct = X::conj(h.tau);
#pragma unroll
      for (int j = k + 1; j < N; ++j) {
        T w = a[k][j];
#pragma unroll
        for (int r = k + 1; r < M; ++r) w = X::cfma(a[r][k], a[r][j], w);
        const T tw = X::mul(ct, w);
        a[k][j] = X::sub(a[k][j], tw);
#pragma unroll
        for (int r = k + 1; r < M; ++r) a[r][j] = X::fnms(a[r][k], tw, a[r][j]);
      }
    }
  }

  static __device__ __forceinline__ void run(const TinyArgs &p) {
    __shared__ __align__(16) float sm[kWarps * kSmemWordsPerWarp];
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    const long long base = ((long long)blockIdx.x * kWarps + warp) * 32;  // first matrix of warp
    if (base >= p.batch) return;
    const long long mat = base + lane;
    const bool active = mat < p.batch;
    T a[M][N];
    T tau[K];
    if (kCanStage && p.staged) {
      float *ws = sm + warp * kSmemWordsPerWarp;
      const float4 *src = reinterpret_cast<const float4 *>(reinterpret_cast<const T *>(p.A) + base * (M * N));
      const long long nmat = min(32LL, p.batch - base);
      const int nchunk = (int)nmat * Q;
#pragma unroll
      for (int s = 0; s < Q; ++s) {
        const int f = lane + 32 * s;
        if (f < nchunk) reinterpret_cast<float4 *>(ws)[swz(f)] = src[f];
      }
      __syncwarp();
#pragma unroll
      for (int c = 0; c < Q; ++c) {
        const float4 v = reinterpret_cast<const float4 *>(ws)[swz(Q * lane + c)];
        const float w4[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const int word = 4 * c + q;        // word index in the column-major matrix
          const int e = word / E, part = word % E;
          const int r = e % M, col = e / M;
          set_word(a[r][col], part, w4[q]);
        }
      }
      factor(a, tau);
      __syncwarp();
#pragma unroll
      for (int c = 0; c < Q; ++c) {
        float w4[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const int word = 4 * c + q;
          const int e = word / E, part = word % E;
          const int r = e % M, col = e / M;
          w4[q] = get_word(a[r][col], part);
        }
        reinterpret_cast<float4 *>(ws)[swz(Q * lane + c)] = make_float4(w4[0], w4[1], w4[2], w4[3]);
      }
      __syncwarp();
      float4 *dst = reinterpret_cast<float4 *>(reinterpret_cast<T *>(p.A) + base * (M * N));
#pragma unroll
      for (int s = 0; s < Q; ++s) {
        const int f = lane + 32 * s;
        if (f < nchunk) dst[f] = reinterpret_cast<const float4 *>(ws)[swz(f)];
      }
    } else {
      const T *Ab = reinterpret_cast<const T *>(p.A) + (active ? mat : base) * (long long)p.lda * N;
#pragma unroll
      for (int j = 0; j < N; ++j)
#pragma unroll
        for (int r = 0; r < M; ++r) a[r][j] = active ? Ab[r + j * p.lda] : X::zero();
      factor(a, tau);
      if (active) {
        T *Aw = reinterpret_cast<T *>(p.A) + mat * (long long)p.lda * N;
#pragma unroll
        for (int j = 0; j < N; ++j)
#pragma unroll
          for (int r = 0; r < M; ++r) Aw[r + j * p.lda] = a[r][j];
      }
    }
    if (active) {
      T *tg = reinterpret_cast<T *>(p.tau) + mat * K;
#pragma unroll
      for (int k = 0; k < K; ++k) tg[k] = tau[k];
    }
  }
};

template <class T, int M, int N>
__global__ void __launch_bounds__(Tiny<T, M, N>::kWarps * 32) geqrf_tiny_kernel(const TinyArgs p) {
  Tiny<T, M, N>::run(p);
}

}  // namespace bqr

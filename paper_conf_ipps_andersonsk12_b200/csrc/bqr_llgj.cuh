// bqr_llgj.cuh -- left-looking register-block Gauss-Jordan without pivoting
// for the GJ56 shape ([A | b], A 56 x 56 fp32, one right-hand side; paper
// Sec. III-B, Fig. 11; NEXT-3).
//
// Arithmetic of bqr_lu.cu's Gauss-Jordan (Listings 5-7): per
// column k the pivot's IEEE reciprocal (0 and info = k+1 for an exactly zero
// pivot; reading L1), row k scaled by it from column k on, and every other
// row updated a_ij -= m_i u_j with the multiplier m_i = a_ik (unscaled; the
// column keeps it, reading L2) and u_j the scaled row k, j > k.
// The ORDER is the left-looking one of bqr_ll.cuh / bqr_lll.cuh: column
// blocks [0,16) [16,32) [32,44) [44,57); only the current block is in
// registers (2 matrices per warp, 4 row lanes x 4 column groups, row pairs
// 8p + 2rg, 8p + 2rg + 1).  An earlier column k reaches the block as: scale
// its row k by 1/pivot_k (kept in shared memory), broadcast it (one shuffle
// per slot), subtract m_k u.  The multiplier columns are full height, so
// they are re-read from the matrix itself (already written back, resident
// in L1/L2) instead of being kept in shared memory; 17 warps = 34 matrices
// per SM.
#pragma once
#include "bqr_common.cuh"

namespace bqr {
namespace llgj {

struct Args {
  float *A;
  float *B;
  int *info;
  long long batch;
  int lda, ldb;
  long long strideA, strideB;
};

constexpr int kN = 56;       // A is kN x kN, b is column kN of [A | b]
constexpr int MP = 7;
constexpr int NSMAX = 4;
constexpr int kWarps = 17;
constexpr int kThreads = 32 * kWarps;
__host__ __device__ constexpr int blk_ns(int b) { return b == 2 ? 3 : 4; }
__host__ __device__ constexpr int blk_c0(int b) { return b == 0 ? 0 : blk_c0(b - 1) + 4 * blk_ns(b - 1); }
constexpr int kNB = 4;
static_assert(blk_c0(kNB - 1) + 4 * blk_ns(kNB - 1) >= kN + 1, "blocks cover [A | b]");
// shared words per matrix: 1/pivot of every column, a two-entry ring of the
// multiplier column (4 row lanes x 14 rows) for the block's own steps
constexpr int kScaleOff = 0;
constexpr int kRingOff = kN;
constexpr int kRingBuf = 4 * 2 * MP;
constexpr int kMatWords = kRingOff + 2 * kRingBuf;  // 168
constexpr size_t kSmemBytes = (size_t)kWarps * 2 * kMatWords * 4;

__device__ __forceinline__ void wsync() { asm volatile("bar.warp.sync -1;" ::: "memory"); }
__device__ __forceinline__ float2 lds64(const float *p) {
  float2 v;
  const unsigned s = (unsigned)__cvta_generic_to_shared(p);
  asm volatile("ld.shared.v2.f32 {%0,%1}, [%2];" : "=f"(v.x), "=f"(v.y) : "r"(s));
  return v;
}

struct Ctx {
  float *sm;
  float *A0;  // this lane's rows (2 rg, 2 rg + 1) of column 0
  float *Bb;  // this lane's rows of b
  int lda;
  int rg, cg, lane;
  int info;
};

using Tile = float2[MP][NSMAX];

// global column c of [A | b] at this lane's rows (nullptr: padding column)
__device__ __forceinline__ float *colp(const Ctx &c, int col) {
  return col < kN ? c.A0 + (long long)col * c.lda : (col == kN ? c.Bb : nullptr);
}

template <int B, int J>
__device__ __forceinline__ void load_slot(const Ctx &c, Tile &a) {
  if constexpr (B < kNB && J < blk_ns(B)) {
    const float *col = colp(c, blk_c0(B) + c.cg + 4 * J);
#pragma unroll
    for (int p = 0; p < MP; ++p) a[p][J] = col ? *reinterpret_cast<const float2 *>(col + 8 * p) : make_float2(0.f, 0.f);
  }
}
template <int B, int J>
__device__ __forceinline__ void store_slot(const Ctx &c, const Tile &a) {
  float *col = colp(c, blk_c0(B) + c.cg + 4 * J);
  if (col) {
#pragma unroll
    for (int p = 0; p < MP; ++p) *reinterpret_cast<float2 *>(col + 8 * p) = a[p][J];
  }
}

// column k's step on slots [J0, J1) of the block: row k scaled by `scale`
// (columns >= k when MASK0: the pivot slot from column group kk on), then
// a -= m u with u the scaled row k (columns > k) and m (zero at row k) at
// mp (shared) or read from global memory (gm)
template <int P, int J0, int J1, bool MASK0>
__device__ __forceinline__ void gj_apply(const Ctx &c, Tile &a, const float2 (&m)[MP], float scale, int kk) {
  if constexpr (J0 < J1) {
    constexpr int NS = J1 - J0, q0 = P / 2;
    const int kr = 4 * (P % 2) + kk;  // row k = 8 q0 + kr
    const bool mine = c.rg == (kr >> 1);
    const int src = (c.lane & ~3) | (kr >> 1);
    float nu[NS];
#pragma unroll
    for (int j = 0; j < NS; ++j) {
      float2 &x = a[q0][J0 + j];
      const bool live = !MASK0 || j > 0 || c.cg >= kk;  // column >= k
      const float xs = ((kr & 1) ? x.y : x.x) * scale;
      if (mine && live) {
        if (kr & 1) x.y = xs; else x.x = xs;
      }
      float u = __shfl_sync(0xffffffffu, xs, src);
      if (MASK0 && j == 0) u = c.cg > kk ? u : 0.f;  // column k keeps its multipliers
      nu[j] = -u;
    }
#pragma unroll
    for (int p = 0; p < MP; ++p)
#pragma unroll
      for (int j = 0; j < NS; ++j) a[p][J0 + j] = __ffma2_rn(m[p], make_float2(nu[j], nu[j]), a[p][J0 + j]);
  }
}

// the multiplier column k (rows of this lane), zero at row k
template <int P>
__device__ __forceinline__ void mult_global(const Ctx &c, float2 (&m)[MP], int kk) {
  const int k = 4 * P + kk;
  const float *col = c.A0 + (long long)k * c.lda;
  const int kr = 4 * (P % 2) + kk;
#pragma unroll
  for (int p = 0; p < MP; ++p) m[p] = *reinterpret_cast<const float2 *>(col + 8 * p);
  if (c.rg == (kr >> 1)) {
    if (kr & 1) m[P / 2].y = 0.f; else m[P / 2].x = 0.f;
  }
}

template <int B, int P>
__device__ __forceinline__ void left(const Ctx &c, Tile &a) {
  if constexpr (P < blk_c0(B) / 4) {
#pragma unroll 1
    for (int kk = 0; kk < 4; ++kk) {
      float2 m[MP];
      mult_global<P>(c, m, kk);
      gj_apply<P, 0, blk_ns(B), false>(c, a, m, c.sm[kScaleOff + 4 * P + kk], kk);
    }
    left<B, P + 1>(c, a);
  }
}

// elimination of block B, panel P (columns 4P .. 4P + 3 in slot s)
template <int B, int P>
__device__ __forceinline__ void panels(Ctx &c, Tile &a) {
  constexpr int P0 = blk_c0(B) / 4, NS = blk_ns(B);
  if constexpr (P < P0 + NS) {
    constexpr int s = P - P0, q0 = P / 2;
    if constexpr (4 * P < kN) {
#pragma unroll 1
      for (int kk = 0; kk < 4; ++kk) {
        const int k = 4 * P + kk;
        const int kr = 4 * (P % 2) + kk;
        const float px = (kr & 1) ? a[q0][s].y : a[q0][s].x;
        const float piv = __shfl_sync(0xffffffffu, px, (c.lane & 16) | (kk * 4) | (kr >> 1));
        const bool z = piv == 0.f;
        const float scale = z ? 0.f : __fdiv_rn(1.0f, piv);
        c.info = (c.info == 0 && z) ? k + 1 : c.info;
        // the multiplier column (owner column group) to the ring, the
        // pivot's reciprocal to the scale list
        float *mp = c.sm + kRingOff + (k & 1) * kRingBuf + c.rg * (2 * MP);
        if (c.cg == kk) {
#pragma unroll
          for (int p = 0; p < MP; ++p) {
            float2 v = a[p][s];
            if (p == q0 && c.rg == (kr >> 1)) {
              if (kr & 1) v.y = 0.f; else v.x = 0.f;
            }
            *reinterpret_cast<float2 *>(mp + 2 * p) = v;
          }
        }
        if ((c.lane & 15) == 0) c.sm[kScaleOff + k] = scale;
        wsync();
        float2 m[MP];
#pragma unroll
        for (int p = 0; p < MP; ++p) m[p] = lds64(mp + 2 * p);
        gj_apply<P, s, NS, true>(c, a, m, scale, kk);
      }
    }
    store_slot<B, s>(c, a);
    load_slot<B + 1, s>(c, a);
    panels<B, P + 1>(c, a);
  }
}

template <int B>
__device__ __forceinline__ void do_block(Ctx &c, Tile &a) {
  if constexpr (B == 0) load_slot<B, 0>(c, a);
  if constexpr (B == 0 || blk_ns(B - 1) <= 1) load_slot<B, 1>(c, a);
  if constexpr (B == 0 || blk_ns(B - 1) <= 2) load_slot<B, 2>(c, a);
  if constexpr (B == 0 || blk_ns(B - 1) <= 3) load_slot<B, 3>(c, a);
  wsync();  // the previous block's columns (multipliers) are in global memory
  left<B, 0>(c, a);
  panels<B, blk_c0(B) / 4>(c, a);
  wsync();
}

__global__ void __launch_bounds__(kThreads, 1) gj_llgj56_kernel(Args args) {
  extern __shared__ float smem_llgj[];
  const int lane = threadIdx.x & 31, warp = __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0);
  const int half = lane >> 4;
  Ctx c;
  c.lane = lane;
  c.rg = lane & 3;
  c.cg = (lane >> 2) & 3;
  c.sm = smem_llgj + (warp * 2 + half) * kMatWords;
  c.lda = args.lda;
  const long long npairs = (args.batch + 1) / 2;
  const long long chunk = (npairs + gridDim.x - 1) / gridDim.x;
  for (long long wq = warp; wq < chunk; wq += kWarps) {
    const long long q = (long long)blockIdx.x * chunk + wq;
    if (q >= npairs) break;
    const long long idx = 2 * q + half;
    const long long mi = idx < args.batch ? idx : idx - 1;  // spare half-warp: same bits, same addresses
    c.A0 = args.A + mi * args.strideA + 2 * c.rg;
    c.Bb = args.B + mi * args.strideB + 2 * c.rg;
    c.info = 0;
    wsync();
    Tile a;
    do_block<0>(c, a);
    do_block<1>(c, a);
    do_block<2>(c, a);
    do_block<3>(c, a);
    if (args.info && (lane & 15) == 0) args.info[mi] = c.info;
    wsync();
  }
}

}  // namespace llgj
}  // namespace bqr

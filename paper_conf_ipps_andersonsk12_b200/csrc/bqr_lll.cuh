// bqr_lll.cuh -- left-looking register-block LU without pivoting for the
// L56 shape (56 x 56 fp32, the paper's 8,000-problem LU comparison, Fig. 11,
// P:L1009; NEXT-3).
//
// Arithmetic of bqr_lu.cu (paper Sec. III-A; Listings 5-7,
// P:L549-593): per column the pivot's IEEE reciprocal (0 and info = k+1 for
// an exactly zero pivot, the elimination continues), l = column * scale
// below the pivot, and the rank-1 update a -= l u with u the pivot row.
// The ORDER is the left-looking one of bqr_ll.cuh (the 56 x 56 QR class):
// column blocks [0,12) [12,24) [24,40) [40,56); only the current block is
// in registers (2 matrices per warp, 4 row lanes x 4 column groups, row
// pairs 8p + 2rg, 8p + 2rg + 1), the earlier blocks' l columns are applied
// to it from shared memory (each needs only row k of the block, which its
// own lane already holds: one shuffle per slot, no reduction), then the
// block is eliminated right-looking.  17 warps = 34 matrices per SM.  Each
// element receives the same fma(-l, u, a) sequence as in the right-looking
// kernel, in the same order of k.
#pragma once
#include "bqr_common.cuh"

namespace bqr {
namespace lll {

struct Args {
  float *A;
  int *info;
  long long batch;
  int lda;
  long long strideA;
};

constexpr int kM = 56;
constexpr int MP = 7;
constexpr int NSMAX = 4;
constexpr int kWarps = 17;
constexpr int kThreads = 32 * kWarps;
__host__ __device__ constexpr int blk_ns(int b) { return b <= 1 ? 3 : 4; }
__host__ __device__ constexpr int blk_c0(int b) { return b == 0 ? 0 : blk_c0(b - 1) + 4 * blk_ns(b - 1); }
constexpr int kNB = 4;
constexpr int kKeepP = 10;  // l columns 0..39 kept for the left-looking applies
__host__ __device__ constexpr int vlen(int P) { return 2 * (MP - P / 2); }
__host__ __device__ constexpr int voff(int P) { return P == 0 ? 0 : voff(P - 1) + 16 * vlen(P - 1); }
constexpr int kVStore = voff(kKeepP);
constexpr int kRingQ = kKeepP / 2;
constexpr int kRingLen = 2 * (MP - kRingQ);
constexpr int kRingBuf = 4 * kRingLen;
constexpr int kMatWords = kVStore + 2 * kRingBuf;  // 1632
constexpr size_t kSmemBytes = (size_t)kWarps * 2 * kMatWords * 4;
static_assert(kSmemBytes <= 232448, "one CTA of 34 matrices per SM");
static_assert(blk_c0(kNB - 1) == 4 * kKeepP && blk_c0(kNB - 1) + 4 * blk_ns(kNB - 1) == kM, "blocks");

__device__ __forceinline__ void wsync() { asm volatile("bar.warp.sync -1;" ::: "memory"); }
__device__ __forceinline__ float2 lds64(const float *p) {
  float2 v;
  const unsigned s = (unsigned)__cvta_generic_to_shared(p);
  asm volatile("ld.shared.v2.f32 {%0,%1}, [%2];" : "=f"(v.x), "=f"(v.y) : "r"(s));
  return v;
}

struct Ctx {
  float *sm;
  float *Ab;  // this lane's element (rows 2 rg, 2 rg + 1; column cg)
  int lda;
  int rg, cg, lane;
  int info;
};

using Tile = float2[MP][NSMAX];

template <int P>
__device__ __forceinline__ float *lptr(const Ctx &c, int kk) {
  if constexpr (P < kKeepP) {
    return c.sm + voff(P) + (kk * 4 + c.rg) * vlen(P);
  } else {
    return c.sm + kVStore + (kk & 1) * kRingBuf + c.rg * kRingLen + (P / 2 - kRingQ) * 2;
  }
}

template <int B, int J>
__device__ __forceinline__ void load_slot(const Ctx &c, Tile &a) {
  if constexpr (B < kNB && J < blk_ns(B)) {
    const float *col = c.Ab + (long long)(blk_c0(B) + 4 * J) * c.lda;
#pragma unroll
    for (int p = 0; p < MP; ++p) a[p][J] = *reinterpret_cast<const float2 *>(col + 8 * p);
  }
}
template <int B, int J>
__device__ __forceinline__ void store_slot(const Ctx &c, const Tile &a) {
  float *col = c.Ab + (long long)(blk_c0(B) + 4 * J) * c.lda;
#pragma unroll
  for (int p = 0; p < MP; ++p) *reinterpret_cast<float2 *>(col + 8 * p) = a[p][J];
}

// a -= l_k u_k on slots [J0, J1): u = row k of each slot (from the lane of
// this column group holding it), l from shared memory (zero at and above
// the pivot); MASK0: the first slot only for columns cg > kk
template <int P, int J0, int J1, bool MASK0>
__device__ __forceinline__ void lapply(const Ctx &c, Tile &a, const float *lp, int kk) {
  if constexpr (J0 < J1) {
    constexpr int NS = J1 - J0, q0 = P / 2;
    const int kr = 4 * (P % 2) + kk;  // row k = 8 q0 + kr
    const int src = (c.lane & ~3) | (kr >> 1);
    float u[NS];
#pragma unroll
    for (int j = 0; j < NS; ++j) {
      const float x = (kr & 1) ? a[q0][J0 + j].y : a[q0][J0 + j].x;
      float y = __shfl_sync(0xffffffffu, x, src);
      if (MASK0 && j == 0) y = c.cg > kk ? y : 0.f;
      u[j] = -y;
    }
#pragma unroll
    for (int p = q0; p < MP; ++p) {
      const float2 l = lds64(lp + 2 * (p - q0));
#pragma unroll
      for (int j = 0; j < NS; ++j) a[p][J0 + j] = __ffma2_rn(l, make_float2(u[j], u[j]), a[p][J0 + j]);
    }
  }
}

template <int B, int P>
__device__ __forceinline__ void left(const Ctx &c, Tile &a) {
  if constexpr (P < blk_c0(B) / 4) {
#pragma unroll 1
    for (int kk = 0; kk < 4; ++kk) lapply<P, 0, blk_ns(B), false>(c, a, lptr<P>(c, kk), kk);
    left<B, P + 1>(c, a);
  }
}

// IEEE reciprocal of the pivot of column kn = 4 PP + kkn (slot S; row kn
// in pair PP/2 of the lane rg = kr/2 of column group kkn), 0 for an exactly
// zero pivot (info = kn + 1 of the first one; reading L1)
template <int PP, int S>
__device__ __forceinline__ float pivot_scale(Ctx &c, const Tile &a, int kkn, int kn) {
  constexpr int q = PP / 2;
  const int kr = 4 * (PP % 2) + kkn;
  const float px = (kr & 1) ? a[q][S].y : a[q][S].x;
  const float piv = __shfl_sync(0xffffffffu, px, (c.lane & 16) | (kkn * 4) | (kr >> 1));
  const bool z = piv == 0.f;
  c.info = (c.info == 0 && z) ? kn + 1 : c.info;
  return z ? 0.f : __fdiv_rn(1.0f, piv);
}

// column k = 4P + kk (slot s): l = a * scale below the pivot, in place and
// to shared memory (owner column group)
template <int P, int S>
__device__ __forceinline__ void publish_l(const Ctx &c, Tile &a, int kk, float scale, float *lp) {
  constexpr int q0 = P / 2;
  const int k = 4 * P + kk;
  const bool own = c.cg == kk;
#pragma unroll
  for (int p = q0; p < MP; ++p) {
    const float2 x = a[p][S];
    const float2 xs = __fmul2_rn(x, make_float2(scale, scale));
    const int r0 = 8 * p + 2 * c.rg;
    float2 l = xs;
    if (p == q0) {
      l.x = r0 > k ? xs.x : 0.f;
      l.y = r0 + 1 > k ? xs.y : 0.f;
    }
    if (own) {
      a[p][S] = p == q0 ? make_float2(r0 > k ? xs.x : x.x, r0 + 1 > k ? xs.y : x.y) : xs;
      *reinterpret_cast<float2 *>(lp + 2 * (p - q0)) = l;
    }
  }
}

// elimination of block B, panel P (columns 4P .. 4P + 3 in slot s), with a
// one-column look-ahead: step k updates the slot holding column k+1 first
// and forms that pivot's reciprocal while the other slots are updated.
// `scale` enters as the reciprocal of column 4P's pivot.
template <int B, int P>
__device__ __forceinline__ void panels(Ctx &c, Tile &a, float scale) {
  constexpr int P0 = blk_c0(B) / 4, NS = blk_ns(B);
  if constexpr (P < P0 + NS) {
    constexpr int s = P - P0;
#pragma unroll 1
    for (int kk = 0; kk < 3; ++kk) {
      const int k = 4 * P + kk;
      float *lp = lptr<P>(c, kk);
      publish_l<P, s>(c, a, kk, scale, lp);
      wsync();
      lapply<P, s, s + 1, true>(c, a, lp, kk);
      scale = pivot_scale<P, s>(c, a, kk + 1, k + 1);
      lapply<P, s + 1, NS, false>(c, a, lp, kk);
    }
    {
      const int k = 4 * P + 3;
      float *lp = lptr<P>(c, 3);
      publish_l<P, s>(c, a, 3, scale, lp);
      wsync();
      if constexpr (s + 1 < NS) {
        lapply<P, s + 1, s + 2, false>(c, a, lp, 3);
        scale = pivot_scale<P + 1, s + 1>(c, a, 0, k + 1);
        lapply<P, s + 2, NS, false>(c, a, lp, 3);
      }
    }
    store_slot<B, s>(c, a);
    load_slot<B + 1, s>(c, a);
    panels<B, P + 1>(c, a, scale);
  }
}

template <int B>
__device__ __forceinline__ void do_block(Ctx &c, Tile &a) {
  if constexpr (B == 0) load_slot<B, 0>(c, a);
  if constexpr (B == 0 || blk_ns(B - 1) <= 1) load_slot<B, 1>(c, a);
  if constexpr (B == 0 || blk_ns(B - 1) <= 2) load_slot<B, 2>(c, a);
  if constexpr (B == 0 || blk_ns(B - 1) <= 3) load_slot<B, 3>(c, a);
  left<B, 0>(c, a);
  const float scale = pivot_scale<blk_c0(B) / 4, 0>(c, a, 0, blk_c0(B));
  panels<B, blk_c0(B) / 4>(c, a, scale);
  wsync();
}

__global__ void __launch_bounds__(kThreads, 1) getrf_lll56_kernel(Args args) {
  extern __shared__ float smem_lll[];
  const int lane = threadIdx.x & 31, warp = __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0);
  const int half = lane >> 4;
  Ctx c;
  c.lane = lane;
  c.rg = lane & 3;
  c.cg = (lane >> 2) & 3;
  c.sm = smem_lll + (warp * 2 + half) * kMatWords;
  c.lda = args.lda;
  const long long npairs = (args.batch + 1) / 2;
  const long long chunk = (npairs + gridDim.x - 1) / gridDim.x;
  for (long long wq = warp; wq < chunk; wq += kWarps) {
    const long long q = (long long)blockIdx.x * chunk + wq;
    if (q >= npairs) break;
    const long long idx = 2 * q + half;
    const long long mi = idx < args.batch ? idx : idx - 1;  // spare half-warp: same bits, same addresses
    c.Ab = args.A + mi * args.strideA + (long long)c.cg * args.lda + 2 * c.rg;
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

}  // namespace lll
}  // namespace bqr

// bqr_ll.cuh -- left-looking register-block Householder QR for the C3
// headline shape (56 x 56 fp32; BASELINE config 3, "5,000
// 56x56 QR factorizations").
//
// Same arithmetic as the right-looking register-file classes (bqr_rf.cuh):
// xLARFG per column (norm, IEEE sqrt/div: "a square root, two divides, and
// two multiplies") and H_k = I - tau_k v_k v_k^T applied as a
// matrix-vector product plus a rank-1 update (Table VI), in the
// paper's 2D-cyclic register layout (Fig. 6) with 4 row lanes x
// 4 column groups per matrix, two matrices per warp.  What changes is the
// ORDER of the column updates (a "blocked algorithm"):
//
//   * the 56 columns are factored in three column blocks [0,20) [20,36)
//     [36,56); only the current block lives in registers (<= 14 rows x 5
//     slots per lane instead of the whole 14 x 14 tile), so the kernel holds
//     17 warps = 34 matrices per SM at <= 120 registers: 5,000 matrices are
//     ONE resident round on 148 SMs (the right-looking class holds 16 per SM
//     at 255 registers: 2.11 rounds, 2 warps per scheduler, IPC 1.6);
//   * a block is loaded from HBM when it is reached, H_0..H_{c0-1} of the
//     earlier blocks are applied to it (left-looking: the reflectors are
//     known, so this is pure matrix-vector/rank-1 throughput with no
//     reflector chain), then it is factored right-looking with a one-column
//     look-ahead (apply H_k to the slot of column k+1, form reflector k+1,
//     apply H_k to the other slots) and written back;
//   * the Householder vectors of the first two blocks stay in shared memory
//     (row-lane-major, rows from the reflector's first live register-row
//     pair, 6.3 KB per matrix) for the later blocks; the last block
//     publishes through a two-entry ring;
//   * packed FP32 (fma.rn.f32x2, SASS FFMA2) on register-row pairs
//     (rows rg + 8p, rg + 8p + 4): v pairs come straight from 8-byte shared
//     loads, so no operand moves are needed.
// Rows of a reflector above its pivot are stored as exact zeros, so the
// applies need no row masks; only the pivot's register row is masked in the
// reflector itself and the pivot slot's columns <= k in the update.
#pragma once
#include "bqr_common.cuh"

namespace bqr {
namespace ll {

struct LlArgs {
  float *A;
  float *tau;
  long long batch;
  int lda;
  long long strideA, strideT;
};

// paired left-looking applies (one reduction for H_k, H_{k+1}): parity
// green but slower on B200 (81.4 vs 69.6 us: 484 B of spills at the
// 96-register cap), off
#ifndef BQR_LL_PAIR
#define BQR_LL_PAIR 0
#endif
constexpr int kM = 56;      // rows = columns
constexpr int MP = 7;       // register-row pairs per lane: rows 8p + 2rg, 8p + 2rg + 1 (8-byte loads)
constexpr int NSMAX = 4;    // column slots per lane of a block (columns c0 + cg + 4j)
constexpr int kWarps = 17;  // one CTA of 17 warps (34 matrices) per SM
constexpr int kThreads = 32 * kWarps;
// column blocks (BQR_LL_PART 0: [0,16) [16,28) [28,40) [40,56);
// 1: [0,8) [8,24) [24,40) [40,56); 2: [0,12) [12,24) [24,40) [40,56))
#ifndef BQR_LL_PART
#define BQR_LL_PART 2
#endif
constexpr int kPart = BQR_LL_PART;
__host__ __device__ constexpr int blk_ns(int b) {
  return kPart == 0 ? (b == 0 ? 4 : (b == 1 ? 3 : (b == 2 ? 3 : 4)))
                    : (kPart == 1 ? (b == 0 ? 2 : 4) : (b <= 1 ? 3 : 4));
}
__host__ __device__ constexpr int blk_c0(int b) { return b == 0 ? 0 : blk_c0(b - 1) + 4 * blk_ns(b - 1); }
constexpr int kNB = 4;
// reflectors of panels 0..9 (columns 0..39) are kept for the left-looking
// applies; panel P's vector holds this lane's pairs P/2 .. MP-1
constexpr int kKeepP = 10;
__host__ __device__ constexpr int vlen(int P) { return 2 * (MP - P / 2); }
__host__ __device__ constexpr int voff(int P) { return P == 0 ? 0 : voff(P - 1) + 16 * vlen(P - 1); }
constexpr int kVStore = voff(kKeepP);       // 1600 words
constexpr int kRingQ = kKeepP / 2;          // first pair of the ring vectors
constexpr int kRingOff = kVStore;           // 2 x [4 row lanes][pairs kRingQ..6]
constexpr int kRingLen = 2 * (MP - kRingQ);
constexpr int kRingBuf = 4 * kRingLen;
constexpr int kTauOff = kRingOff + 2 * kRingBuf;
// g_k = v_{k+1}^T v_k for the reflector pairs (k, k+1), k even < 4 kKeepP,
// of the paired left-looking applies
constexpr int kGOff = kTauOff + kM;
constexpr int kMatWords = kGOff + (BQR_LL_PAIR ? 2 * kKeepP : 0);  // 1688 (1708) words: 34 matrices = 224 (227) KB
constexpr size_t kSmemBytes = (size_t)kWarps * 2 * kMatWords * 4;
static_assert(NSMAX == 4, "do_block loads slots 0..3");
static_assert(kMatWords % 2 == 0, "8-byte aligned vectors");
static_assert(kSmemBytes <= 232448, "one CTA of 34 matrices per SM");
static_assert(blk_c0(kNB - 1) == 4 * kKeepP && blk_c0(kNB - 1) + 4 * blk_ns(kNB - 1) == kM, "blocks");

// packed FP32 (one fma.rn.f32x2 per row pair) or two scalar FMAs: on B200
// one warp issues an FFMA2 every ~2.8 cycles but a 3-register FFMA every
// ~1.1 (tools/micro/ffma2_rate.cu: 23 vs 29 FMA/clk per scheduler), so for
// a latency-bound warp the scalar form is faster
#ifndef BQR_LL_FFMA2
#define BQR_LL_FFMA2 1
#endif
__device__ __forceinline__ float2 fma2(float2 a, float2 b, float2 c) {
#if BQR_LL_FFMA2
  return __ffma2_rn(a, b, c);
#else
  return make_float2(fmaf(a.x, b.x, c.x), fmaf(a.y, b.y, c.y));
#endif
}

__device__ __forceinline__ void wsync() { asm volatile("bar.warp.sync -1;" ::: "memory"); }
__device__ __forceinline__ float2 lds64(const float *p) {
  float2 v;
  const unsigned s = (unsigned)__cvta_generic_to_shared(p);
  asm volatile("ld.shared.v2.f32 {%0,%1}, [%2];" : "=f"(v.x), "=f"(v.y) : "r"(s));
  return v;
}

#ifdef BQR_LL_TIMING
// debug builds only: clock64 stamps of CTA 0's warps (first matrix pair):
// [warp][event], events 3B = block B start, 3B+1 after its left-looking
// applies, 3B+2 after its panels, 12 = end of the matrix
constexpr int kDbgEv = 13;
static __device__ unsigned long long g_ll_dbg[kWarps * kDbgEv];
#define LL_STAMP(c, e)                                                              \
  do {                                                                              \
    if (blockIdx.x == 0 && (c).lane == 0 && (c).first) g_ll_dbg[(threadIdx.x >> 5) * kDbgEv + (e)] = clock64(); \
  } while (0)
#else
#define LL_STAMP(c, e) \
  do {                 \
  } while (0)
#endif

struct Ctx {
  float *sm;    // this matrix's shared words
  float *Ab;    // this lane's element (rg, cg) of the matrix in global memory
  int lda;
  int rg, cg, lane;
#ifdef BQR_LL_TIMING
  bool first;
#endif
};

// this lane's vector of reflector k = 4P + kk, positioned at pair P/2
template <int P>
__device__ __forceinline__ float *vptr(const Ctx &c, int kk) {
  if constexpr (P < kKeepP) {
    return c.sm + voff(P) + (kk * 4 + c.rg) * vlen(P);
  } else {
    return c.sm + kRingOff + (kk & 1) * kRingBuf + c.rg * kRingLen + (P / 2 - kRingQ) * 2;
  }
}

using Tile = float2[MP][NSMAX];

// unroll of the left-looking reflector loop.  1 keeps the kernel at 5.3k
// SASS instructions (9.2k at 4): the same full-batch time (69.8 us), but a
// cold instruction cache after the L2 flush costs a lone warp 25 us less
// (batch 1: 30.8 vs 62.4 us; batch 625: 32.8 vs 54.3 us)
#ifndef BQR_LL_UNROLL_LEFT
#define BQR_LL_UNROLL_LEFT 1
#endif
constexpr int kUnrollLeft = BQR_LL_UNROLL_LEFT;
// one butterfly for the look-ahead dot and the next column's norm
// (apply1_look / reflector_fused): parity green but slower on B200 (79.4 vs
// 69.7 us: 100 B of spills at the 96-register cap, 15% more code), off
#ifndef BQR_LL_FUSED
#define BQR_LL_FUSED 0
#endif
#ifndef BQR_LL_LOADLAG
#define BQR_LL_LOADLAG 0
#endif
#ifndef BQR_LL_PACKRED
#define BQR_LL_PACKRED 1
#endif

// slot j of block B (columns c0 + cg + 4j, rows rg + 4i) <-> HBM
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


// H_k = I - tau v v^T on slots [J0, J1), rows from pair Q0 (v is zero above
// its pivot); MASK0: slot J0 only for the columns cg > kk (pivot slot)
template <int Q0, int J0, int J1, bool MASK0>
__device__ __forceinline__ void apply(const Ctx &c, Tile &a, const float *vp, float tau, int kk) {
  if constexpr (J0 < J1) {
    constexpr int NS = J1 - J0;
    float2 v[MP];
#pragma unroll
    for (int p = Q0; p < MP; ++p) v[p] = lds64(vp + 2 * (p - Q0));
    float2 w[NS];
#pragma unroll
    for (int j = 0; j < NS; ++j) w[j] = make_float2(0.f, 0.f);
#pragma unroll
    for (int p = Q0; p < MP; ++p)
#pragma unroll
      for (int j = 0; j < NS; ++j) w[j] = fma2(v[p], a[p][J0 + j], w[j]);
    float2 nt[NS];
#if BQR_LL_PACKRED
    // column pairs packed for the FP32 pipe: (w_j.x + w_j.y, w_j+1.x + w_j+1.y)
    // as one FADD2, the butterfly adds as FADD2, -tau * s as FMUL2
    constexpr int NP = (NS + 1) / 2;
    float2 sp[NP];
#pragma unroll
    for (int q = 0; q < NP; ++q) {
      if (2 * q + 1 < NS)
        sp[q] = __fadd2_rn(make_float2(w[2 * q].x, w[2 * q + 1].x), make_float2(w[2 * q].y, w[2 * q + 1].y));
      else
        sp[q] = make_float2(w[2 * q].x + w[2 * q].y, 0.f);
    }
#pragma unroll
    for (int o = 1; o <= 2; o <<= 1) {
#pragma unroll
      for (int q = 0; q < NP; ++q) {
        if (2 * q + 1 < NS) {
          const float2 r = make_float2(__shfl_xor_sync(0xffffffffu, sp[q].x, o), __shfl_xor_sync(0xffffffffu, sp[q].y, o));
          sp[q] = __fadd2_rn(sp[q], r);
        } else {
          sp[q].x += __shfl_xor_sync(0xffffffffu, sp[q].x, o);
        }
      }
    }
#pragma unroll
    for (int q = 0; q < NP; ++q) {
      const float2 t = __fmul2_rn(sp[q], make_float2(-tau, -tau));
      float t0 = t.x;
      if (MASK0 && q == 0) t0 = c.cg > kk ? t0 : 0.f;
      nt[2 * q] = make_float2(t0, t0);
      if (2 * q + 1 < NS) nt[2 * q + 1] = make_float2(t.y, t.y);
    }
#else
    float s[NS];
#pragma unroll
    for (int j = 0; j < NS; ++j) s[j] = w[j].x + w[j].y;
#pragma unroll
    for (int j = 0; j < NS; ++j) s[j] += __shfl_xor_sync(0xffffffffu, s[j], 1);
#pragma unroll
    for (int j = 0; j < NS; ++j) s[j] += __shfl_xor_sync(0xffffffffu, s[j], 2);
#pragma unroll
    for (int j = 0; j < NS; ++j) {
      float t = tau * s[j];
      if (MASK0 && j == 0) t = c.cg > kk ? t : 0.f;
      nt[j] = make_float2(-t, -t);
    }
#endif
#pragma unroll
    for (int p = Q0; p < MP; ++p)
#pragma unroll
      for (int j = 0; j < NS; ++j) a[p][J0 + j] = fma2(v[p], nt[j], a[p][J0 + j]);
  }
}

// xLARFG of column kn = 4 PP + kkn held in slot S (computed by every lane;
// the owner column group cg == kkn uses it)
template <int PP, int S>
__device__ __forceinline__ Reflector<float> reflector(const Ctx &c, const Tile &a, int kkn) {
  constexpr int q0 = PP / 2;
  float2 acc[2] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
  float alpha = 0.f;
#pragma unroll
  for (int p = q0; p < MP; ++p) {
    float2 x = a[p][S];
    if (p == q0) {
      // pair q0 holds rows 8 q0 + 2 rg (x) and + 1 (y); the pivot is row
      // 8 q0 + kr
      const int kr = 4 * (PP % 2) + kkn;
      alpha = 2 * c.rg == kr ? x.x : (2 * c.rg + 1 == kr ? x.y : 0.f);
      x.x = 2 * c.rg > kr ? x.x : 0.f;
      x.y = 2 * c.rg + 1 > kr ? x.y : 0.f;
    }
    acc[(p - q0) & 1] = fma2(x, x, acc[(p - q0) & 1]);
  }
  const float2 accs = __fadd2_rn(acc[0], acc[1]);
  float sig = accs.x + accs.y;
  sig += __shfl_xor_sync(0xffffffffu, sig, 1);
  sig += __shfl_xor_sync(0xffffffffu, sig, 2);
  alpha = __shfl_sync(0xffffffffu, alpha, (c.lane & ~3) | ((4 * (PP % 2) + kkn) >> 1));
  return make_reflector(alpha, sig);
}

// owner lanes: v = x * scal below the pivot, 1 at it, 0 above; the column
// becomes [R; V] (beta at the pivot); v and tau go to shared memory.
// Non-owner lanes multiply by 1 (bit-exact no-op), branch-free.
template <int PP, int S>
__device__ __forceinline__ void publish(const Ctx &c, Tile &a, const Reflector<float> &h, int kkn, float *vdst,
                                        float *tslot) {
  constexpr int q0 = PP / 2;
  const bool own = c.cg == kkn;
  const float scal = own ? h.scal : 1.f;
#pragma unroll
  for (int p = q0; p < MP; ++p) {
    const float2 x = a[p][S];
    const float2 xs = __fmul2_rn(x, make_float2(scal, scal));
    float2 v = xs, nx = xs;
    if (p == q0) {
      const int kr = 4 * (PP % 2) + kkn, r0 = 2 * c.rg, r1 = 2 * c.rg + 1;
      v.x = r0 > kr ? xs.x : (r0 == kr ? 1.f : 0.f);
      nx.x = r0 > kr ? xs.x : ((own && r0 == kr) ? h.beta : x.x);
      v.y = r1 > kr ? xs.y : (r1 == kr ? 1.f : 0.f);
      nx.y = r1 > kr ? xs.y : ((own && r1 == kr) ? h.beta : x.y);
    }
    a[p][S] = nx;
    if (own) *reinterpret_cast<float2 *>(vdst + 2 * (p - q0)) = v;
  }
  if (own && c.rg == 0) *tslot = h.tau;
}

// ---------------------------------------------------------------- fused look-ahead
// H_k on the single slot S holding column k+1, returning alongside the dot
// gamma = sum_{r >= k} a_r^2 of this lane's column BEFORE the update (one
// butterfly for both): H_k is orthogonal on rows >= k, so after it the
// squared norm below row k+1 is gamma - a'_k^2 - a'_{k+1}^2 (reflector_fused)
template <int Q0, int S, bool MASK0>
__device__ __forceinline__ float apply1_look(const Ctx &c, Tile &a, const float *vp, float tau, int kk, int k) {
  float2 v[MP];
#pragma unroll
  for (int p = Q0; p < MP; ++p) v[p] = lds64(vp + 2 * (p - Q0));
  float2 w = make_float2(0.f, 0.f), g = make_float2(0.f, 0.f);
#pragma unroll
  for (int p = Q0; p < MP; ++p) {
    w = fma2(v[p], a[p][S], w);
    float2 x = a[p][S];
    if (p == Q0) {
      const int r0 = 8 * p + 2 * c.rg;
      x.x = r0 >= k ? x.x : 0.f;
      x.y = r0 + 1 >= k ? x.y : 0.f;
    }
    g = fma2(x, x, g);
  }
  float sd = w.x + w.y, gg = g.x + g.y;
  sd += __shfl_xor_sync(0xffffffffu, sd, 1);
  gg += __shfl_xor_sync(0xffffffffu, gg, 1);
  sd += __shfl_xor_sync(0xffffffffu, sd, 2);
  gg += __shfl_xor_sync(0xffffffffu, gg, 2);
  float t = tau * sd;
  if (MASK0) t = c.cg > kk ? t : 0.f;
  const float2 nt = make_float2(-t, -t);
#pragma unroll
  for (int p = Q0; p < MP; ++p) a[p][S] = fma2(v[p], nt, a[p][S]);
  return gg;
}

// xLARFG of column kn = 4 PP + kkn (slot S) from gamma: sigma = gamma -
// a'_{kn-1}^2 - alpha^2, accurate while it cancels at most one bit; a
// warp-uniform fallback to the direct norm (reflector) otherwise, which also
// keeps tau = 0 exact for an already triangular column (reading Q5)
template <int PP, int S>
__device__ __forceinline__ Reflector<float> reflector_fused(const Ctx &c, const Tile &a, int kkn, float gam) {
  const int kn = 4 * PP + kkn, k = kn - 1;
  constexpr int qn = PP / 2;
  // pair of row k: qn, or the previous pair when kn opens an even panel
  const int krow = k & 7, knrow = kn & 7;
  float xk_own, xa_own;
  {
    const float2 pn = a[qn][S];
    xa_own = (knrow & 1) ? pn.y : pn.x;
    if constexpr (PP % 2 == 0 && qn > 0) {
      const float2 pk = kkn == 0 ? a[qn - 1][S] : pn;
      xk_own = (krow & 1) ? pk.y : pk.x;
    } else {
      xk_own = (krow & 1) ? pn.y : pn.x;
    }
  }
  const float xk = __shfl_sync(0xffffffffu, xk_own, (c.lane & ~3) | (krow >> 1));
  const float xa = __shfl_sync(0xffffffffu, xa_own, (c.lane & ~3) | (knrow >> 1));
  const float nu2 = fmaf(-xk, xk, gam);
  const float sig = fmaf(-xa, xa, nu2);
  const bool own = c.cg == kkn;
  const bool bad = own && !(nu2 >= 0.5f * gam && sig >= 0.0625f * nu2);
  if (__any_sync(0xffffffffu, bad)) return reflector<PP, S>(c, a, kkn);
  return make_reflector(xa, sig);
}

// ---------------------------------------------------------------- phases
// left-looking: H_0 .. H_{c0-1} (panels 0 .. c0/4 - 1) on block B
// H_{k+1} H_k on slots [0, NS) in one pass (k even, both of panel P, rows
// from pair Q0): with w = v_k^T A, w' = v_{k+1}^T A (ONE reduction for both)
// and g = v_{k+1}^T v_k, H_{k+1} H_k A = A - v_k t^T - v_{k+1} t'^T where
// t = tau_k w and t' = tau_{k+1} (w' - g t)
template <int Q0, int NS>
__device__ __forceinline__ void apply_pair(const Ctx &c, Tile &a, const float *vp0, const float *vp1, float tau0,
                                           float tau1, float g) {
  float2 w0[NS], w1[NS];
#pragma unroll
  for (int j = 0; j < NS; ++j) w0[j] = w1[j] = make_float2(0.f, 0.f);
#pragma unroll
  for (int p = Q0; p < MP; ++p) {
    const float2 v0 = lds64(vp0 + 2 * (p - Q0)), v1 = lds64(vp1 + 2 * (p - Q0));
#pragma unroll
    for (int j = 0; j < NS; ++j) {
      w0[j] = fma2(v0, a[p][j], w0[j]);
      w1[j] = fma2(v1, a[p][j], w1[j]);
    }
  }
  float2 sp[NS];  // (v_k^T a_j, v_{k+1}^T a_j)
#pragma unroll
  for (int j = 0; j < NS; ++j)
    sp[j] = __fadd2_rn(make_float2(w0[j].x, w1[j].x), make_float2(w0[j].y, w1[j].y));
#pragma unroll
  for (int o = 1; o <= 2; o <<= 1)
#pragma unroll
    for (int j = 0; j < NS; ++j)
      sp[j] = __fadd2_rn(sp[j], make_float2(__shfl_xor_sync(0xffffffffu, sp[j].x, o),
                                            __shfl_xor_sync(0xffffffffu, sp[j].y, o)));
  float2 n0[NS], n1[NS];
#pragma unroll
  for (int j = 0; j < NS; ++j) {
    const float t0 = tau0 * sp[j].x;
    const float t1 = tau1 * fmaf(-g, t0, sp[j].y);
    n0[j] = make_float2(-t0, -t0);
    n1[j] = make_float2(-t1, -t1);
  }
#pragma unroll
  for (int p = Q0; p < MP; ++p) {
    const float2 v0 = lds64(vp0 + 2 * (p - Q0)), v1 = lds64(vp1 + 2 * (p - Q0));
#pragma unroll
    for (int j = 0; j < NS; ++j) a[p][j] = fma2(v1, n1[j], fma2(v0, n0[j], a[p][j]));
  }
}

template <int B, int P>
__device__ __forceinline__ void left(const Ctx &c, Tile &a) {
  if constexpr (P < blk_c0(B) / 4) {
    const float *taus = c.sm + kTauOff;
#if BQR_LL_PAIR
#pragma unroll
    for (int kk = 0; kk < 4; kk += 2)
      apply_pair<P / 2, blk_ns(B)>(c, a, vptr<P>(c, kk), vptr<P>(c, kk + 1), taus[4 * P + kk], taus[4 * P + kk + 1],
                                   c.sm[kGOff + 2 * P + kk / 2]);
#else
#pragma unroll kUnrollLeft
    for (int kk = 0; kk < 4; ++kk) apply<P / 2, 0, blk_ns(B), false>(c, a, vptr<P>(c, kk), taus[4 * P + kk], kk);
#endif
    left<B, P + 1>(c, a);
  }
}

// g_k = v_{k+1}^T v_k of the pairs (k, k+1) of panel P (k = 4P, 4P + 2),
// written by lane (rg 0, cg 0) of the matrix
template <int P>
__device__ __forceinline__ void gram_pairs(const Ctx &c) {
  constexpr int Q0 = P / 2;
#pragma unroll
  for (int kk = 0; kk < 4; kk += 2) {
    const float *vp0 = vptr<P>(c, kk), *vp1 = vptr<P>(c, kk + 1);
    float2 acc = make_float2(0.f, 0.f);
#pragma unroll
    for (int p = Q0; p < MP; ++p) acc = fma2(lds64(vp0 + 2 * (p - Q0)), lds64(vp1 + 2 * (p - Q0)), acc);
    float g = acc.x + acc.y;
    g += __shfl_xor_sync(0xffffffffu, g, 1);
    g += __shfl_xor_sync(0xffffffffu, g, 2);
    if (c.rg == 0 && c.cg == 0) c.sm[kGOff + 2 * P + kk / 2] = g;
  }
}
template <int P, int PE>
__device__ __forceinline__ void gram_block(const Ctx &c) {
  if constexpr (P < PE && P < kKeepP) {
    gram_pairs<P>(c);
    gram_block<P + 1, PE>(c);
  }
}

// right-looking factorisation of block B, panel P (slot s = P - c0/4), with
// the one-column look-ahead; reflector 4P is published on entry
template <int B, int P>
__device__ __forceinline__ void panels(const Ctx &c, Tile &a) {
  constexpr int P0 = blk_c0(B) / 4, NS = blk_ns(B);
  if constexpr (P < P0 + NS) {
    constexpr int s = P - P0, q0 = P / 2;
    float *taus = c.sm + kTauOff;
#pragma unroll 1
    for (int kk = 0; kk < 3; ++kk) {
      wsync();
      const int k = 4 * P + kk;
      const float tau = taus[k];
      const float *vp = vptr<P>(c, kk);
#if BQR_LL_FUSED
      const float gam = apply1_look<q0, s, true>(c, a, vp, tau, kk, k);
      const Reflector<float> h = reflector_fused<P, s>(c, a, kk + 1, gam);
#else
      apply<q0, s, s + 1, true>(c, a, vp, tau, kk);
      const Reflector<float> h = reflector<P, s>(c, a, kk + 1);
#endif
      apply<q0, s + 1, NS, false>(c, a, vp, tau, kk);
      publish<P, s>(c, a, h, kk + 1, vptr<P>(c, kk + 1), taus + k + 1);
    }
    // slot s is final: write it back and start loading slot s of the next
    // block into the same registers (its latency hides behind the rest of
    // this block)
    store_slot<B, s>(c, a);
#if BQR_LL_LOADLAG
    // one panel later: the store has read the registers by then (no WAR
    // stall of the load behind the store queue)
    if constexpr (s >= 1) load_slot<B + 1, s - 1>(c, a);
    if constexpr (s + 1 == NS) load_slot<B + 1, s>(c, a);
#else
    load_slot<B + 1, s>(c, a);
#endif
    if constexpr (s + 1 < NS) {
      wsync();
      const int k = 4 * P + 3;
      const float tau = taus[k];
      const float *vp = vptr<P>(c, 3);
#if BQR_LL_FUSED
      const float gam = apply1_look<q0, s + 1, false>(c, a, vp, tau, 3, k);
      const Reflector<float> h = reflector_fused<P + 1, s + 1>(c, a, 0, gam);
#else
      apply<q0, s + 1, s + 2, false>(c, a, vp, tau, 3);
      const Reflector<float> h = reflector<P + 1, s + 1>(c, a, 0);
#endif
      apply<q0, s + 2, NS, false>(c, a, vp, tau, 3);
      publish<P + 1, s + 1>(c, a, h, 0, vptr<P + 1>(c, 0), taus + k + 1);
    }
    panels<B, P + 1>(c, a);
  }
}

template <int B>
__device__ __forceinline__ void do_block(const Ctx &c, Tile &a) {
  constexpr int P0 = blk_c0(B) / 4;
  // slots beyond the previous block's width (all of block 0) load here; the
  // others were loaded while the previous block finished
  LL_STAMP(c, 3 * B);
  if constexpr (B == 0) load_slot<B, 0>(c, a);
  if constexpr (B == 0 || blk_ns(B - 1) <= 1) load_slot<B, 1>(c, a);
  if constexpr (B == 0 || blk_ns(B - 1) <= 2) load_slot<B, 2>(c, a);
  if constexpr (B == 0 || blk_ns(B - 1) <= 3) load_slot<B, 3>(c, a);
  left<B, 0>(c, a);
  LL_STAMP(c, 3 * B + 1);
  {
    // head reflector of the block (column c0, slot 0)
    const Reflector<float> h = reflector<P0, 0>(c, a, 0);
    publish<P0, 0>(c, a, h, 0, vptr<P0>(c, 0), c.sm + kTauOff + 4 * P0);
  }
  panels<B, P0>(c, a);
  wsync();
#if BQR_LL_PAIR
  // the pair products g of this block's reflectors, for the later blocks
  gram_block<P0, P0 + blk_ns(B)>(c);
  wsync();
#endif
  LL_STAMP(c, 3 * B + 2);
}

__global__ void __launch_bounds__(kThreads, 1) geqrf_ll56_kernel(LlArgs args) {
  extern __shared__ float smem_ll[];
  // the warp index through a shuffle: provably warp-uniform, so the matrix
  // loop below is a uniform branch (otherwise ptxas guards every later
  // shuffle with a divergence check, BRA.DIV, that splits the basic blocks
  // the scheduler interleaves the reflector chain across)
  const int lane = threadIdx.x & 31, warp = __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0);
  const int half = lane >> 4;
  Ctx c;
  c.lane = lane;
  c.rg = lane & 3;
  c.cg = (lane >> 2) & 3;
  c.sm = smem_ll + (warp * 2 + half) * kMatWords;
#ifdef BQR_LL_TIMING
  c.first = true;
#endif
  const long long npairs = (args.batch + 1) / 2;
  // CTA b owns the contiguous pairs [b chunk, (b + 1) chunk), chunk =
  // ceil(pairs / grid) with grid = min(pairs, SMs): a full batch gives 17
  // pairs per SM as before, a batch smaller than one resident round spreads
  // over all SMs (one warp per SM first) instead of filling few SMs
  const long long chunk = (npairs + gridDim.x - 1) / gridDim.x;
  for (long long wq = warp; wq < chunk; wq += kWarps) {
    const long long q = (long long)blockIdx.x * chunk + wq;
    if (q >= npairs) break;
    const long long idx = 2 * q + half;
    // odd batch: the spare half-warp factors its neighbour's matrix again
    // with the same instructions on the same data, so its stores write the
    // same bits to the same addresses (no divergent branch around them)
    const long long mi = idx < args.batch ? idx : idx - 1;
    wsync();
    c.Ab = args.A + mi * args.strideA + (long long)c.cg * args.lda + 2 * c.rg;
    c.lda = args.lda;
    Tile a;
    do_block<0>(c, a);
    do_block<1>(c, a);
    do_block<2>(c, a);
    do_block<3>(c, a);
    {
      const float *taus = c.sm + kTauOff;
      float *tg = args.tau + mi * args.strideT;
#pragma unroll
      for (int t = lane & 15; t < kM; t += 16) tg[t] = taus[t];
    }
    wsync();
    LL_STAMP(c, 12);
#ifdef BQR_LL_TIMING
    c.first = false;
#endif
  }
}

}  // namespace ll
}  // namespace bqr

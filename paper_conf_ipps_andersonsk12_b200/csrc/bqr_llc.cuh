// bqr_llc.cuh -- left-looking register-block complex Householder QR for the
// STAP headline shape (240 x 66 complex64, optionally with the right-hand
// side b as column 66 of [A | b]: the fused Q^H b of P:L313; BASELINE
// config 4, Sec. VII).
//
// Arithmetic: ZGEQR2 order -- per column the reflector (ZLARFG: norm, IEEE
// sqrt/div) and H_k^H = I - conj(tau_k) v_k v_k^H applied as a
// matrix-vector product plus a rank-1 update (Table VI) -- in the
// paper's 2D-cyclic register layout (Fig. 6): 8 row lanes x 4
// column groups per warp, 6 warps = 24 column groups per CTA; element (r, c)
// lives in lane (r mod 8, c mod 24), register (r div 8, c div 24).
//
// B200 design (see bqr_ll.cuh for the real 56 x 56 counterpart): the
// right-looking class keeps the whole 240 x 67 tile in registers, one
// matrix per SM, so 256 matrices take 1.73 rounds of a latency-bound
// CTA.  Here the columns are factored in three blocks of 24, [0,24)
// [24,48) [48,67): only the current block is in registers (30 rows x one
// slot per lane); a block is loaded when it is reached, H_0..H_{c0-1} are
// applied to it from shared memory (left-looking; no reflector chain), then
// it is factored right-looking.  The 48 Householder vectors of the first two
// blocks stay in shared memory (86 KB), so TWO matrices fit per SM (2 x 6
// warps, 2 x 90 KB): 256 matrices are one resident round on 148 SMs.
// Packed FP32 (fma.rn.f32x2) on the (re, im) pair with v as the broadcast
// scalar operand; vectors live in shared memory as 16-byte chunks of two
// rows, chunk-major so the 8 row lanes read consecutive chunks.
#pragma once
#include "bqr_common.cuh"

namespace bqr {
namespace llc {

struct Args {
  float2 *A;
  float2 *tau;
  float2 *B;
  long long batch;
  int lda, ldb, nrhs;
  long long strideA, strideT, strideB;
};

constexpr int kM = 240, kN = 66;
constexpr int R = 8, MR = 30;          // row lanes; rows rg + 8 i, i < 30
constexpr int kWarps = 6, G = 4 * kWarps;  // 24 column groups
constexpr int kThreads = 32 * kWarps;
constexpr int NSMAX = 1;
constexpr int kNB = 3;
// column blocks [0,24) [24,48) [48,72): one slot (24 columns) per lane
__host__ __device__ constexpr int blk_c0(int b) { return 24 * b; }
__host__ __device__ constexpr int blk_ns(int) { return 1; }
constexpr int kKeepP = 6;  // row panels (8 columns each) of block 0: reflectors 0..47 kept
// 16-byte chunks (two rows) per row lane of a reflector of row panel P
__host__ __device__ constexpr int chunks(int P) { return (MR - P + 1) / 2; }
__host__ __device__ constexpr int voff(int P) { return P == 0 ? 0 : voff(P - 1) + 8 * R * chunks(P - 1); }
constexpr int kVStore = voff(kKeepP);          // float4 units
constexpr int kRingChunks = chunks(kKeepP);    // >= chunks of every later panel
constexpr int kRingOff = kVStore;
constexpr int kRingBuf = kRingChunks * R;
constexpr int kTauOff = kRingOff + 2 * kRingBuf;  // float4 units; 72 float2 taus follow
constexpr size_t kSmemBytes = (size_t)kTauOff * 16 + 72 * 8;
static_assert(kSmemBytes * 2 <= 228 * 1024 - 2048, "two CTAs per SM");

__device__ __forceinline__ float4 lds128(const float4 *p) {
  float4 v;
  const unsigned s = (unsigned)__cvta_generic_to_shared(p);
  asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(s));
  return v;
}
__device__ __forceinline__ void bsync() { asm volatile("bar.sync 0;" ::: "memory"); }

struct Ctx {
  float4 *vs;    // vector store (float4 chunks)
  float2 *taus;  // [72]
  int rg, cg, lane, warp;
  float2 *Ab;    // this lane's row rg of the matrix (column 0)
  float2 *Bb;    // this lane's row rg of the right-hand side, or null
  int lda;
};

using Tile = float2[MR][NSMAX];

// this lane's chunk 0 of reflector k = 8P + kk (rows 8P + rg, 8P + 8 + rg, ...)
template <int P>
__device__ __forceinline__ float4 *vptr(const Ctx &c, int kk) {
  if constexpr (P < kKeepP) {
    return c.vs + voff(P) + kk * R * chunks(P) + c.rg;
  } else {
    return c.vs + kRingOff + (kk & 1) * kRingBuf + c.rg;
  }
}

__device__ __forceinline__ float2 f2(float x, float y) { return make_float2(x, y); }

// H_k^H on slots [J0, J1), rows from register row P (v zero above its pivot):
// w = v^H a (reduced over the 8 row lanes), a -= v (conj(tau) w); MASK0: the
// first slot only for columns cg > kkg (the pivot slot; kkg = pivot's group)
template <int P, int J0, int J1, bool MASK0>
__device__ __forceinline__ void apply(const Ctx &c, Tile &a, const float4 *vp, float2 ct, int kkg) {
  if constexpr (J0 < J1) {
    constexpr int NS = J1 - J0;
    constexpr int NQ = chunks(P);
    float2 wa[NS][2], wb[NS][2];
#pragma unroll
    for (int j = 0; j < NS; ++j) wa[j][0] = wa[j][1] = wb[j][0] = wb[j][1] = f2(0.f, 0.f);
#pragma unroll
    for (int q = 0; q < NQ; ++q) {
      const float4 f = lds128(vp + q * R);
      const int i = P + 2 * q;
#pragma unroll
      for (int j = 0; j < NS; ++j) {
        wa[j][0] = __ffma2_rn(f2(f.x, f.x), a[i][J0 + j], wa[j][0]);
        wb[j][0] = __ffma2_rn(f2(f.y, f.y), a[i][J0 + j], wb[j][0]);
        if (i + 1 < MR) {
          wa[j][1] = __ffma2_rn(f2(f.z, f.z), a[i + 1][J0 + j], wa[j][1]);
          wb[j][1] = __ffma2_rn(f2(f.w, f.w), a[i + 1][J0 + j], wb[j][1]);
        }
      }
    }
    float2 t[NS];
#pragma unroll
    for (int j = 0; j < NS; ++j) {
      const float2 A2 = __fadd2_rn(wa[j][0], wa[j][1]), B2 = __fadd2_rn(wb[j][0], wb[j][1]);
      float2 s = f2(A2.x + B2.y, A2.y - B2.x);  // conj(v)^T a
#pragma unroll
      for (int o = 1; o < R; o <<= 1)
        s = __fadd2_rn(s, f2(__shfl_xor_sync(0xffffffffu, s.x, o), __shfl_xor_sync(0xffffffffu, s.y, o)));
      // t = conj(tau) * s
      float2 tt = f2(fmaf(ct.x, s.x, -ct.y * s.y), fmaf(ct.x, s.y, ct.y * s.x));
      if (MASK0 && j == 0) tt = c.cg > kkg ? tt : f2(0.f, 0.f);
      t[j] = tt;
    }
#pragma unroll
    for (int q = 0; q < NQ; ++q) {
      const float4 f = lds128(vp + q * R);
      const int i = P + 2 * q;
#pragma unroll
      for (int j = 0; j < NS; ++j) {
        const float2 n1 = f2(-t[j].x, -t[j].y), n2 = f2(t[j].y, -t[j].x);
        a[i][J0 + j] = __ffma2_rn(f2(f.y, f.y), n2, __ffma2_rn(f2(f.x, f.x), n1, a[i][J0 + j]));
        if (i + 1 < MR)
          a[i + 1][J0 + j] = __ffma2_rn(f2(f.w, f.w), n2, __ffma2_rn(f2(f.z, f.z), n1, a[i + 1][J0 + j]));
      }
    }
  }
}

// ZLARFG of column kn = 8 P + kr in slot S (owner lanes: cg == group of kn)
template <int P, int S>
__device__ __forceinline__ Reflector<float2> reflector(const Ctx &c, const Tile &a, int kr) {
  float2 acc[2] = {f2(0.f, 0.f), f2(0.f, 0.f)};
  float2 alpha = f2(0.f, 0.f);
#pragma unroll
  for (int i = P; i < MR; ++i) {
    float2 x = a[i][S];
    if (i == P) {
      alpha = c.rg == kr ? x : f2(0.f, 0.f);
      x = c.rg > kr ? x : f2(0.f, 0.f);
    }
    acc[(i - P) & 1] = __ffma2_rn(x, x, acc[(i - P) & 1]);
  }
  const float2 s2 = __fadd2_rn(acc[0], acc[1]);
  float sig = s2.x + s2.y;
#pragma unroll
  for (int o = 1; o < R; o <<= 1) sig += __shfl_xor_sync(0xffffffffu, sig, o);
  const int src = (c.lane & ~(R - 1)) | kr;
  alpha = f2(__shfl_sync(0xffffffffu, alpha.x, src), __shfl_sync(0xffffffffu, alpha.y, src));
  return make_reflector(alpha, sig);
}

// owner lanes (cg == kg): v = x scal below the pivot, 1 at it, 0 above; the
// column becomes [R; V] (beta at the pivot); v and tau go to shared memory
template <int P, int S>
__device__ __forceinline__ void publish(const Ctx &c, Tile &a, const Reflector<float2> &hh, int kr, int kg,
                                        float4 *vdst, float2 *tslot) {
  const bool own = c.cg == kg;
  constexpr int NQ = chunks(P);
#pragma unroll
  for (int q = 0; q < NQ; ++q) {
    float2 v[2];
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int i = P + 2 * q + h;
      if (i >= MR) {
        v[h] = f2(0.f, 0.f);
        continue;
      }
      const float2 x = a[i][S];
      const float2 xs = f2(fmaf(x.x, hh.scal.x, -x.y * hh.scal.y), fmaf(x.x, hh.scal.y, x.y * hh.scal.x));
      if (i == P) {
        v[h] = c.rg > kr ? xs : (c.rg == kr ? f2(1.f, 0.f) : f2(0.f, 0.f));
        if (own) a[i][S] = c.rg > kr ? xs : (c.rg == kr ? f2(hh.beta, 0.f) : x);
      } else {
        v[h] = xs;
        if (own) a[i][S] = xs;
      }
    }
    if (own) vdst[q * R] = make_float4(v[0].x, v[0].y, v[1].x, v[1].y);
  }
  if (own && c.rg == 0) *tslot = hh.tau;
}

// ---------------------------------------------------------------- phases
template <int B, int J>
__device__ __forceinline__ void load_slot(const Ctx &c, Tile &a) {
  if constexpr (J < blk_ns(B)) {
    const int col = blk_c0(B) + c.cg + G * J;
    const float2 *p = col < kN ? c.Ab + (long long)col * c.lda : c.Bb;
    const bool live = col < kN || (col == kN && c.Bb != nullptr);
#pragma unroll
    for (int i = 0; i < MR; ++i) a[i][J] = live ? p[8 * i] : f2(0.f, 0.f);
  }
}
template <int B, int J>
__device__ __forceinline__ void store_slot(const Ctx &c, const Tile &a) {
  if constexpr (J < blk_ns(B)) {
    const int col = blk_c0(B) + c.cg + G * J;
    float2 *p = col < kN ? c.Ab + (long long)col * c.lda : c.Bb;
    if (col < kN || (col == kN && c.Bb != nullptr)) {
#pragma unroll
      for (int i = 0; i < MR; ++i) p[8 * i] = a[i][J];
    }
  }
}

// left-looking: H_0 .. H_{c0-1} (row panels 0 .. c0/8 - 1) on block B
template <int B, int P>
__device__ __forceinline__ void left(const Ctx &c, Tile &a) {
  if constexpr (P < blk_c0(B) / 8) {
#pragma unroll 2
    for (int kk = 0; kk < 8; ++kk) {
      const float2 tau = c.taus[8 * P + kk];
      apply<P, 0, blk_ns(B), false>(c, a, vptr<P>(c, kk), f2(tau.x, -tau.y), 0);
    }
    left<B, P + 1>(c, a);
  }
}

// right-looking factorisation of block B, row panel P (columns 8P .. 8P+7,
// slot s = (8P - c0) / 24); reflector 8P is published on entry.  Step k:
// the warp owning column k+1 applies H_k to that slot first, forms and
// publishes reflector k+1, then applies H_k to the rest; other warps apply
// H_k to their live slots; one CTA barrier per column.
template <int B, int P>
__device__ __forceinline__ void panels(const Ctx &c, Tile &a) {
  constexpr int c0 = blk_c0(B), NS = blk_ns(B);
  constexpr int P0 = c0 / 8, PE = (c0 + G * NS) / 8;
  if constexpr (P < PE && 8 * P < kN) {
    constexpr int s = (8 * P - c0) / G;
    constexpr int kg0 = (8 * P - c0) % G;  // group of column 8P
    constexpr int kend = (8 * P + 8 < kN ? 8 * P + 8 : kN) - 8 * P;
#pragma unroll 1
    for (int kk = 0; kk < kend; ++kk) {
      bsync();
      const int k = 8 * P + kk;
      const float2 tau = c.taus[k];
      const float2 ct = f2(tau.x, -tau.y);
      const float4 *vp = vptr<P>(c, kk);
      const int kn = k + 1;
      if (kk + 1 < 8) {
        // column k+1 in this panel and slot
        const int kgn = kg0 + kk + 1;
        if (kn < kN && c.warp == kgn / 4) {
          apply<P, s, s + 1, true>(c, a, vp, ct, kg0 + kk);
          const Reflector<float2> h = reflector<P, s>(c, a, kk + 1);
          publish<P, s>(c, a, h, kk + 1, kgn, vptr<P>(c, kk + 1), c.taus + kn);
          apply<P, s + 1, NS, false>(c, a, vp, ct, 0);
        } else {
          // a warp whose four column groups are all factored (<= the
          // pivot's group) has nothing left in this block's slot
          if (4 * c.warp + 3 > kg0 + kk) apply<P, s, NS, true>(c, a, vp, ct, kg0 + kk);
        }
      } else {
        // column k+1 opens row panel P+1 (maybe the next slot)
        constexpr int sn = (8 * P + 8 - c0) / G, kgn = (8 * P + 8 - c0) % G;
        if (kn < kN && sn < NS && c.warp == kgn / 4) {
          if constexpr (sn < NS) {
            apply<P, s, s + 1, true>(c, a, vp, ct, kg0 + kk);
            if constexpr (sn != s) apply<P, sn, sn + 1, false>(c, a, vp, ct, 0);
            const Reflector<float2> h = reflector<P + 1, sn>(c, a, 0);
            publish<P + 1, sn>(c, a, h, 0, kgn, vptr<P + 1>(c, 0), c.taus + kn);
            apply<P, sn + 1, NS, false>(c, a, vp, ct, 0);
          }
        } else {
          // a warp whose four column groups are all factored (<= the
          // pivot's group) has nothing left in this block's slot
          if (4 * c.warp + 3 > kg0 + kk) apply<P, s, NS, true>(c, a, vp, ct, kg0 + kk);
        }
      }
    }
    panels<B, P + 1>(c, a);
  }
}

template <int B>
__device__ __forceinline__ void do_block(const Ctx &c, Tile &a) {
  constexpr int P0 = blk_c0(B) / 8;
  load_slot<B, 0>(c, a);
  left<B, 0>(c, a);
  // head reflector of the block (column c0: slot 0, group 0)
  if (c.warp == 0) {
    const Reflector<float2> h = reflector<P0, 0>(c, a, 0);
    publish<P0, 0>(c, a, h, 0, 0, vptr<P0>(c, 0), c.taus + 8 * P0);
  }
  panels<B, P0>(c, a);
  store_slot<B, 0>(c, a);
  bsync();
}

__global__ void __launch_bounds__(kThreads, 2) geqrf_llc240_kernel(Args args) {
  extern __shared__ __align__(16) float4 smem_llc[];
  const int t = threadIdx.x;
  Ctx c;
  c.lane = t & 31;
  c.warp = __shfl_sync(0xffffffffu, t >> 5, 0);
  c.rg = c.lane & (R - 1);
  c.cg = 4 * c.warp + (c.lane >> 3);
  c.vs = smem_llc;
  c.taus = reinterpret_cast<float2 *>(smem_llc + kTauOff);
  c.lda = args.lda;
#pragma unroll 1
  for (long long mat = blockIdx.x; mat < args.batch; mat += gridDim.x) {
    c.Ab = args.A + mat * args.strideA + c.rg;
    c.Bb = args.nrhs > 0 ? args.B + mat * args.strideB + c.rg : nullptr;
    Tile a;
    do_block<0>(c, a);
    do_block<1>(c, a);
    do_block<2>(c, a);
    float2 *tg = args.tau + mat * args.strideT;
    for (int i = t; i < kN; i += kThreads) tg[i] = c.taus[i];
    bsync();
  }
}

}  // namespace llc
}  // namespace bqr

// bqr_llc.cuh -- left-looking register-block complex Householder QR for the
// STAP headline shape (240 x 66 complex64, optionally with the right-hand
// side b as column 66 of [A | b]: the fused Q^H b of P:L313; BASELINE
// config 4, Sec. VII).
//
// Arithmetic: ZGEQR2 order -- per column the reflector (ZLARFG: norm, IEEE
// sqrt/div) and H_k^H = I - conj(tau_k) v_k v_k^H applied as a
// matrix-vector product plus a rank-1 update (Table VI) -- in the
// paper's 2D-cyclic register layout (Fig. 6): a warp is one
// column group (rows lane + 32 i, i < 8), 6 warps per CTA; element (r, c)
// lives in lane r mod 32 of warp c mod 6, register (r div 32, c div 6).
//
// B200 design (bqr_ll.cuh is the real 56 x 56 counterpart): the
// right-looking class keeps the whole 240 x 67 tile in registers, one
// matrix per SM, so 256 matrices take 1.73 rounds.  Here the columns are
// factored in two blocks of 36, [0,36) and [36,67): only the current block
// is in registers (8 rows x 6 slots per lane); block 1 is loaded when block
// 0 is done, H_0..H_35 are applied to it from shared memory (left-looking,
// no reflector chain), then it is factored right-looking.  The 36 vectors of
// block 0 stay in shared memory (72 KB), block 1 publishes through a ring
// of 9, so TWO matrices fit per SM (2 x 6 warps, 2 x 92 KB) and 256 are one
// resident round.  Every reflector has a "full" mbarrier: a warp waits only
// for the vector it is about to apply (no per-column CTA rendezvous); the
// ring is never overwritten while read because warp w publishes every 6th
// column and must have applied every earlier vector first (lag <= G + 2).
// Packed FP32 (fma.rn.f32x2) on the (re, im) pair with v as the broadcast
// scalar operand; vectors as 16-byte chunks of two rows, chunk-major so the
// 32 lanes read 512 contiguous bytes.
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
constexpr int R = 32, MR = 8;          // rows lane + 32 i, i < 8 (rows >= 240 are zero)
constexpr int kWarps = 6, G = kWarps;  // a warp is a column group
constexpr int kThreads = 32 * kWarps;
constexpr int NS = 6;                  // slots per lane: a block is 36 columns
constexpr int kNB = 2;
constexpr int kBW = G * NS;            // block width
__host__ __device__ constexpr int blk_c0(int b) { return kBW * b; }
constexpr int kKeep = kBW;             // reflectors of block 0, kept
constexpr int kChunks = 4;             // 16-byte chunks (2 rows) per lane and vector
constexpr int kVec = kChunks * R;      // float4 per vector (2 KB)
constexpr int kRing = G + 3;           // ring depth for the reflectors of block 1
constexpr int kRingOff = kKeep * kVec;
constexpr int kTauOff = kRingOff + kRing * kVec;  // float4 units: 72 float2 taus
constexpr int kBarOff = kTauOff + 36;             // float4 units: 72 mbarriers
constexpr size_t kSmemBytes = (size_t)kBarOff * 16 + 72 * 8;
static_assert(2 * (kSmemBytes + 1024) <= 228 * 1024, "two CTAs per SM");
// first register row of the vectors of 6-column group S6 (its first column / 32)
__host__ __device__ constexpr int row0(int S6) { return (G * S6) / R; }
static_assert(row0((kN - 1) / G) <= 2 && row0(kKeep / G - 1) == 0, "chunk layout");

__device__ __forceinline__ float4 lds128(const float4 *p) {
  float4 v;
  const unsigned s = (unsigned)__cvta_generic_to_shared(p);
  asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(s));
  return v;
}
__device__ __forceinline__ unsigned su32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ bool mbar_try(const unsigned long long *bar, unsigned parity) {
  unsigned ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
      "selp.u32 %0, 1, 0, p;\n}"
      : "=r"(ok)
      : "r"(su32(bar)), "r"(parity), "r"(1000000u)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void wsync() { asm volatile("bar.warp.sync -1;" ::: "memory"); }

#ifdef BQR_LLC_TIMING
// debug builds only: clock64 of CTA 0's first matrix, [warp][k][0] = wait for
// v_k returned, [warp][k][1] = v_{k+1} published (its owner), [warp][70..72]
// = block 0 start, block 1 start (before its loads), after block 1's left
static __device__ unsigned long long g_llc_dbg[kWarps * 74 * 2];
#define LLC_STAMP(c, k, e)                                                                   \
  do {                                                                                        \
    if (blockIdx.x == 0 && (c).lane == 0 && (c).first) g_llc_dbg[((c).warp * 74 + (k)) * 2 + (e)] = clock64(); \
  } while (0)
#else
#define LLC_STAMP(c, k, e) \
  do {                     \
  } while (0)
#endif

struct Ctx {
  float4 *vs;
  float2 *taus;
  unsigned long long *full;  // [72]
  unsigned parity;
  int lane, warp;
  float2 *Ab;  // this lane's row of column 0
  float2 *Bb;  // this lane's row of the right-hand side, or null
  int lda;
#ifdef BQR_LLC_TIMING
  bool first;
#endif
};

using Tile = float2[MR][NS];

// lazy rest-update of the next-but-one owner: parity green but slower on
// B200 (134 vs 119 us; a lone matrix 119.6 vs 113 us), off
#ifndef BQR_LLC_LAZY
#define BQR_LLC_LAZY 0
#endif

__device__ __forceinline__ float4 *vptr(const Ctx &c, int k) {
  return c.vs + (k < kKeep ? k * kVec : kRingOff + ((k - kKeep) % kRing) * kVec) + c.lane;
}
__device__ __forceinline__ void wait_full(const Ctx &c, int k) {
  while (!mbar_try(c.full + k, c.parity)) {
  }
}
__device__ __forceinline__ float2 f2(float x, float y) { return make_float2(x, y); }

// H_k^H on slots [J0, J1) of this warp, rows from register row I0 (v is zero
// above its pivot): w = v^H a (butterfly over the 32 lanes), a -= v conj(tau) w
template <int I0, int J0, int J1>
__device__ __forceinline__ void apply3(Tile &a, const float4 *vp, float2 ct) {
  if constexpr (J0 < J1) {
    constexpr int N = J1 - J0;
    float2 wa[N], wb[N];
#pragma unroll
    for (int j = 0; j < N; ++j) wa[j] = wb[j] = f2(0.f, 0.f);
#pragma unroll
    for (int q = 0; q < kChunks; ++q) {
      const int i = I0 + 2 * q;
      if (i < MR) {
        const float4 f = lds128(vp + q * R);
#pragma unroll
        for (int j = 0; j < N; ++j) {
          wa[j] = __ffma2_rn(a[i][J0 + j], f2(f.x, f.x), wa[j]);
          wb[j] = __ffma2_rn(a[i][J0 + j], f2(f.y, f.y), wb[j]);
          if (i + 1 < MR) {
            wa[j] = __ffma2_rn(a[i + 1][J0 + j], f2(f.z, f.z), wa[j]);
            wb[j] = __ffma2_rn(a[i + 1][J0 + j], f2(f.w, f.w), wb[j]);
          }
        }
      }
    }
    float2 t[N];
#pragma unroll
    for (int j = 0; j < N; ++j) {
      float2 s = f2(wa[j].x + wb[j].y, wa[j].y - wb[j].x);  // sum conj(v) a
#pragma unroll
      for (int o = 1; o < R; o <<= 1)
        s = __fadd2_rn(s, f2(__shfl_xor_sync(0xffffffffu, s.x, o), __shfl_xor_sync(0xffffffffu, s.y, o)));
      t[j] = f2(fmaf(ct.x, s.x, -ct.y * s.y), fmaf(ct.x, s.y, ct.y * s.x));
    }
#pragma unroll
    for (int q = 0; q < kChunks; ++q) {
      const int i = I0 + 2 * q;
      if (i < MR) {
        const float4 f = lds128(vp + q * R);
#pragma unroll
        for (int j = 0; j < N; ++j) {
          const float2 n1 = f2(-t[j].x, -t[j].y), n2 = f2(t[j].y, -t[j].x);
          a[i][J0 + j] = __ffma2_rn(f2(f.y, f.y), n2, __ffma2_rn(f2(f.x, f.x), n1, a[i][J0 + j]));
          if (i + 1 < MR)
            a[i + 1][J0 + j] = __ffma2_rn(f2(f.w, f.w), n2, __ffma2_rn(f2(f.z, f.z), n1, a[i + 1][J0 + j]));
        }
      }
    }
  }
}
// slots [J0, J1) in passes of at most three (bounds the live accumulators)
template <int I0, int J0, int J1>
__device__ __forceinline__ void apply(Tile &a, const float4 *vp, float2 ct) {
  if constexpr (J0 < J1) {
    constexpr int JM = J0 + 3 < J1 ? J0 + 3 : J1;
    apply3<I0, J0, JM>(a, vp, ct);
    apply<I0, JM, J1>(a, vp, ct);
  }
}

// ZLARFG of column kn held in slot S of this (owner) warp, rows from I0;
// then the column becomes [R; V] and v_kn, tau_kn are published
template <int I0, int S>
__device__ __forceinline__ void reflect_publish(const Ctx &c, Tile &a, int kn) {
  float2 acc = f2(0.f, 0.f);
  float2 alpha = f2(0.f, 0.f);
#pragma unroll
  for (int i = I0; i < MR; ++i) {
    const int r = c.lane + R * i;
    float2 x = a[i][S];
    alpha = r == kn ? x : alpha;
    x = r > kn ? x : f2(0.f, 0.f);
    acc = __ffma2_rn(x, x, acc);
  }
  float sig = acc.x + acc.y;
#pragma unroll
  for (int o = 1; o < R; o <<= 1) sig += __shfl_xor_sync(0xffffffffu, sig, o);
  const int src = kn & (R - 1);
  alpha = f2(__shfl_sync(0xffffffffu, alpha.x, src), __shfl_sync(0xffffffffu, alpha.y, src));
  const Reflector<float2> h = make_reflector(alpha, sig);
  float4 *vd = vptr(c, kn);
#pragma unroll
  for (int q = 0; q < kChunks; ++q) {
    float2 v[2];
#pragma unroll
    for (int e = 0; e < 2; ++e) {
      const int i = I0 + 2 * q + e;
      if (i >= MR) {
        v[e] = f2(0.f, 0.f);
        continue;
      }
      const int r = c.lane + R * i;
      const float2 x = a[i][S];
      const float2 xs = f2(fmaf(x.x, h.scal.x, -x.y * h.scal.y), fmaf(x.x, h.scal.y, x.y * h.scal.x));
      v[e] = r > kn ? xs : (r == kn ? f2(1.f, 0.f) : f2(0.f, 0.f));
      a[i][S] = r > kn ? xs : (r == kn ? f2(h.beta, 0.f) : x);
    }
    vd[q * R] = make_float4(v[0].x, v[0].y, v[1].x, v[1].y);
  }
  if (c.lane == 0) c.taus[kn] = h.tau;
  LLC_STAMP(c, kn, 1);
  wsync();  // lane 0's tau store before every lane's release
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(c.full + kn)) : "memory");
}

// ---------------------------------------------------------------- phases
template <int B>
__device__ __forceinline__ void load_block(const Ctx &c, Tile &a) {
#pragma unroll
  for (int j = 0; j < NS; ++j) {
    const int col = blk_c0(B) + c.warp + G * j;
    const bool live = col < kN || (col == kN && c.Bb != nullptr);
    const float2 *p = col < kN ? c.Ab + (long long)col * c.lda : c.Bb;
#pragma unroll
    for (int i = 0; i < MR; ++i) a[i][j] = (live && c.lane + R * i < kM) ? p[R * i] : f2(0.f, 0.f);
  }
}
template <int B>
__device__ __forceinline__ void store_block(const Ctx &c, const Tile &a) {
#pragma unroll
  for (int j = 0; j < NS; ++j) {
    const int col = blk_c0(B) + c.warp + G * j;
    const bool live = col < kN || (col == kN && c.Bb != nullptr);
    float2 *p = col < kN ? c.Ab + (long long)col * c.lda : c.Bb;
#pragma unroll
    for (int i = 0; i < MR; ++i)
      if (live && c.lane + R * i < kM) p[R * i] = a[i][j];
  }
}

// left-looking: H_0 .. H_{c0-1} (vectors from register row 0) on every slot
template <int B>
__device__ __forceinline__ void left(const Ctx &c, Tile &a) {
#pragma unroll 1
  for (int k = 0; k < blk_c0(B); ++k) {
    wait_full(c, k);
    const float2 tau = c.taus[k];
    apply<0, 0, NS>(a, vptr(c, k), f2(tau.x, -tau.y));
  }
}

// right-looking factorisation of block B, slot S (columns c0 + 6S + w):
// step k = c0 + 6S + kk waits for v_k; the owner of column k+1 applies H_k
// to the slot holding it, publishes reflector k+1, then applies H_k to its
// other live slots; every other warp applies H_k to its live slots (its
// slot S only if its column there is > k)
template <int B, int S>
__device__ __forceinline__ void panels(const Ctx &c, Tile &a) {
  if constexpr (S < NS) {
    constexpr int c0 = blk_c0(B), S6 = (c0 / G) + S, I0 = row0(S6);
    constexpr int I0p = S > 0 ? row0(S6 - 1) : I0;  // rows of the previous slot's vectors
    constexpr int kbeg = c0 + G * S;
    constexpr int kend = kbeg + G < kN ? kbeg + G : kN;
    constexpr int klim = c0 + kBW < kN ? c0 + kBW : kN;  // pivots of this block: k < klim
#pragma unroll 1
    for (int k = kbeg; k < kend; ++k) {
      const int kk = k - kbeg;
      wait_full(c, k);
      LLC_STAMP(c, k, 0);
      const float2 tau = c.taus[k];
      const float2 ct = f2(tau.x, -tau.y);
      const float4 *vp = vptr(c, k);
      const int kn = k + 1, kn2 = k + 2;
#if BQR_LLC_LAZY
      // lazy rest-update (the right-looking class's LAZY scheme): the owner of
      // column k+2 applies H_k only to the slot holding k+2 and defers its
      // other slots to step k+1, after it has published v_{k+2}; otherwise
      // that rest-update sits between v_{k+1} arriving and its own chain
      const bool o1 = kn < klim && c.warp == (kk + 1) % G;
      const bool o2 = !o1 && kn2 < klim && c.warp == (kk + 2) % G;
      if (o1) {
        const float2 tp = k > c0 ? c.taus[k - 1] : f2(0.f, 0.f);
        const float2 ctp = f2(tp.x, -tp.y);
        const float4 *vpp = vptr(c, k > c0 ? k - 1 : k);
        if (kk + 1 < G) {
          apply<I0, S, S + 1>(a, vp, ct);
          reflect_publish<I0, S>(c, a, kn);
          if (k > c0) {
            if (kk == 0)
              apply<I0p, S + 1, NS>(a, vpp, ctp);
            else
              apply<I0, S + 1, NS>(a, vpp, ctp);
          }
          apply<I0, S + 1, NS>(a, vp, ct);
        } else if constexpr (S + 1 < NS) {
          apply<I0, S + 1, S + 2>(a, vp, ct);
          reflect_publish<row0(S6 + 1), S + 1>(c, a, kn);
          if (k > c0) apply<I0, S + 2, NS>(a, vpp, ctp);
          apply<I0, S + 2, NS>(a, vp, ct);
        }
      } else if (o2) {
        if (kk + 2 < G) {
          apply<I0, S, S + 1>(a, vp, ct);
        } else {
          apply<I0, S + 1, S + 2>(a, vp, ct);
        }
      } else if (c.warp > kk) {
        apply<I0, S, NS>(a, vp, ct);
      } else {
        apply<I0, S + 1, NS>(a, vp, ct);
      }
#else
      if (kk + 1 < G) {
        if (kn < kN && c.warp == kk + 1) {
          apply<I0, S, S + 1>(a, vp, ct);
          reflect_publish<I0, S>(c, a, kn);
          apply<I0, S + 1, NS>(a, vp, ct);
        } else if (c.warp > kk) {
          apply<I0, S, NS>(a, vp, ct);
        } else {
          apply<I0, S + 1, NS>(a, vp, ct);
        }
      } else {
        // column k+1 opens slot S+1 (owner: warp 0), unless the block ends
        if constexpr (S + 1 < NS) {
          if (kn < kN && c.warp == 0) {
            apply<I0, S + 1, S + 2>(a, vp, ct);
            reflect_publish<row0(S6 + 1), S + 1>(c, a, kn);
            apply<I0, S + 2, NS>(a, vp, ct);
          } else {
            apply<I0, S + 1, NS>(a, vp, ct);
          }
        }
      }
#endif
    }
    panels<B, S + 1>(c, a);
  }
}

template <int B>
__device__ __forceinline__ void do_block(const Ctx &c, Tile &a) {
  LLC_STAMP(c, 70 + B, 0);
  load_block<B>(c, a);
  left<B>(c, a);
  LLC_STAMP(c, 72 + B, 0);
  if (c.warp == 0) reflect_publish<row0(blk_c0(B) / G), 0>(c, a, blk_c0(B));
  panels<B, 0>(c, a);
  store_block<B>(c, a);
}

__global__ void __launch_bounds__(kThreads, 2) geqrf_llc240_kernel(Args args) {
  extern __shared__ __align__(16) float4 smem_llc[];
  const int t = threadIdx.x;
  Ctx c;
  c.lane = t & 31;
  c.warp = __shfl_sync(0xffffffffu, t >> 5, 0);
  c.vs = smem_llc;
  c.taus = reinterpret_cast<float2 *>(smem_llc + kTauOff);
  c.full = reinterpret_cast<unsigned long long *>(smem_llc + kBarOff);
  c.lda = args.lda;
  if (t < kN) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(c.full + t)), "r"(32) : "memory");
  }
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncthreads();
  c.parity = 0;
#ifdef BQR_LLC_TIMING
  c.first = true;
#endif
#pragma unroll 1
  for (long long mat = blockIdx.x; mat < args.batch; mat += gridDim.x) {
    c.Ab = args.A + mat * args.strideA + c.lane;
    c.Bb = args.nrhs > 0 ? args.B + mat * args.strideB + c.lane : nullptr;
    Tile a;
    do_block<0>(c, a);
    do_block<1>(c, a);
    __syncthreads();  // every vector consumed, every tau published
    float2 *tg = args.tau + mat * args.strideT;
    for (int i = t; i < kN; i += kThreads) tg[i] = c.taus[i];
    __syncthreads();
    c.parity ^= 1u;
#ifdef BQR_LLC_TIMING
    c.first = false;
#endif
  }
}

}  // namespace llc
}  // namespace bqr

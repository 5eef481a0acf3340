// bqr_rf.cuh -- register-file Householder QR, one matrix per thread group.
//
// The paper's "one problem per block" (Sec. V) keeps the
// whole matrix in the register file in a 2D-cyclic layout (Fig. 6,
// P:L443-499) and, per column, forms the Householder vector with a column
// norm + sqrt/divides by one thread, broadcasts it through shared memory,
// then does a matrix-vector product with a reduction and a rank-1 update
// (Listings 4-7; Table VI).
//
// B200 re-design (not a port):
//   * a "group" of R x G threads owns one matrix; rows are cyclic over the R
//     lanes of a warp segment (so every column reduction -- the norm and the
//     matrix-vector product -- is a warp-shuffle butterfly, no barrier, no
//     thread-0 serial loop) and columns are cyclic over the G column groups;
//     R and G need not be equal (the paper needed p = sqrt(p)^2);
//   * a group is a sub-warp (several matrices per warp, e.g. 2 x 56x56 fp32
//     per warp), a warp, or a CTA (e.g. 240x66 c64 over 11 warps);
//   * look-ahead: inside step k the column group that owns column k+1 first
//     applies H_k to that column, forms reflector k+1 (norm, IEEE sqrt/div)
//     and only then applies H_k to its other columns, so the serial
//     reflector chain overlaps independent FMAs instead of idling the SM;
//     the new vector is published into the other half of a double-buffered
//     shared-memory slot, so ONE group barrier per column suffices;
//   * the compile-time panel recursion advances the first live
//     register row/column slot per panel, so finished rows/columns cost
//     nothing; inside a panel the column loop is a runtime loop (small code);
//   * Householder vectors live in shared memory row-lane-major, so every
//     lane re-reads its rows with 16-byte loads instead of holding them in
//     registers (the matrix itself needs the register file);
//   * global <-> register staging either directly (row lanes >= 8: each warp
//     access is a contiguous column segment) or through a shared-memory tile
//     filled by 16-byte cp.async (small R).
#pragma once
#include "bqr_common.cuh"


namespace bqr {

#ifdef BQR_PHASE_TIMING
// Debug build only (-DBQR_PHASE_TIMING): clock64 stamps of the first matrix
// of CTA 0, [step][warp][phase]: 0 step entry, 1 after the step wait,
// 2 after the look-ahead reflector (owner) / slot P, 3 step end.
constexpr int kDbgSteps = 300, kDbgWarps = 32;
static __device__ unsigned long long g_bqr_dbg[kDbgSteps * kDbgWarps * 4];  // per TU
#define BQR_STAMP(c, k, ph)                                                                \
  do {                                                                                     \
    if ((c).dbg && ((c).lane == 0) && (k) < kDbgSteps)                                     \
      g_bqr_dbg[(((k) * kDbgWarps) + ((c).t >> 5)) * 4 + (ph)] = clock64();                 \
  } while (0)
#else
#define BQR_STAMP(c, k, ph) \
  do {                      \
  } while (0)
#endif

struct RfArgs {
  void *A;
  void *tau;
  long long batch;
  int lda, m, n, kmax;
  int ldS;        // staging tile leading dimension (elements)
  int tileWords;  // staging tile stride per group (32-bit words)
  int vec4;       // 16-byte vectorised staging legal (lda%4==0, m%4==0, aligned)
  int bulk;       // contiguous matrices (lda == m), 16-byte aligned, size % 16 == 0:
                  // stage with one TMA bulk copy per matrix each way
  // augmented right-hand sides (the paper's [A | b]): columns
  // n .. n+nrhs-1 of the register tile are B; they are updated by every
  // reflector but never become pivots, so they end as Q^H B.  Direct
  // (non-staged) kernels only; nrhs = 0 otherwise.
  void *B;
  int ldb, nrhs;
  // batch strides in elements (A, tau, B); LAPACK-contiguous batches use
  // lda*n, kmax, ldb*nrhs; the tiled oversize path passes panel views
  long long strideA, strideT, strideB;
};

// Warp barrier as opaque PTX: nvcc versions the whole rest of a kernel on
// "was the warp diverged at this __syncwarp()" (BRA.DIV + a full copy of the
// factorisation); the asm form keeps one copy.
__device__ __forceinline__ void warp_sync() { asm volatile("bar.warp.sync -1;" ::: "memory"); }

template <int GT, int GPB>
__device__ __forceinline__ void group_sync(int grp) {
  if constexpr (GT <= 32) {
    warp_sync();
  } else if constexpr (GPB == 1) {
    __syncthreads();
  } else {
    asm volatile("bar.sync %0, %1;" ::"r"(8 + grp), "r"(GT) : "memory");
  }
}

// Producer/consumer step barrier of a multi-warp group: the warp that
// publishes reflector k arrives (release, no wait) on named barrier
// 1 + k % NB; every other warp syncs on it before reading the vector.  A
// warp can run ahead only through the steps whose columns it owns itself
// (at most 32/R in a row), so NB = 32/R + 2 rotating IDs (and as many vector
// buffers) keep an early arrival off an instance that has not completed.
template <int GT, int NB>
__device__ __forceinline__ void step_arrive(int k) {
  warp_sync();
  if constexpr (GT > 32) asm volatile("bar.arrive %0, %1;" ::"r"(1 + k % NB), "r"(GT) : "memory");
}
template <int GT, int NB>
__device__ __forceinline__ void step_wait(int k) {
  if constexpr (GT <= 32) {
    warp_sync();
  } else {
    asm volatile("bar.sync %0, %1;" ::"r"(1 + k % NB), "r"(GT) : "memory");
  }
}

__device__ __forceinline__ void cp_async16(void *smem_dst, const void *gmem_src) {
  unsigned s = (unsigned)__cvta_generic_to_shared(smem_dst);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem_src) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;\n" ::: "memory"); }

// TMA bulk copies (cp.async.bulk) completing on an mbarrier / bulk group.
__device__ __forceinline__ unsigned smem_u32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(void *bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void bulk_load(void *dst, const void *src, unsigned bytes, void *bar) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}
// One bounded hardware wait (suspend-time hint); the retry loop is plain
// C++ so the compiler sees structured control flow (an asm-internal branch
// makes it assume the warp may stay diverged and duplicate the whole kernel
// behind a BRA.DIV).
__device__ __forceinline__ bool mbar_try_wait(void *bar, unsigned parity) {
  unsigned ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
      "selp.u32 %0, 1, 0, p;\n}"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity), "r"(1000000u)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void bulk_store(void *dst, const void *src, unsigned bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_u32(src)), "r"(bytes)
               : "memory");
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
__device__ __forceinline__ void bulk_store_drain() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

// 16-byte shared loads that the compiler may not merge across passes (keeps
// the Householder vector out of the register file between the
// matrix-vector product and the rank-1 update).
__device__ __forceinline__ float4 lds128(const void *p) {
  float4 v;
  unsigned s = (unsigned)__cvta_generic_to_shared(p);
  asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(s));
  return v;
}
__device__ __forceinline__ float lds32(const void *p) {
  float v;
  unsigned s = (unsigned)__cvta_generic_to_shared(p);
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(s));
  return v;
}
__device__ __forceinline__ float2 lds64(const void *p) {
  float2 v;
  unsigned s = (unsigned)__cvta_generic_to_shared(p);
  asm volatile("ld.shared.v2.f32 {%0,%1}, [%2];" : "=f"(v.x), "=f"(v.y) : "r"(s));
  return v;
}

template <class T, int R, int G, int MR, int NC, int GPB, bool STAGE, bool EX = false>
struct RfCfg {
  static constexpr int GT = R * G;
  static constexpr int NT = GT * GPB;
  static constexpr int MMAX = R * MR;
  static constexpr int NMAX = G * NC;
  static constexpr int E = sizeof(T) / 4;     // 32-bit words per element
  static constexpr int VW = 4 / E;            // elements per 16-byte vector
  // row-lane-major vector buffer: rows of lane rg at [rg*MRP, rg*MRP+MR);
  // MRP*E == 4 (mod 32) spreads the R lanes over distinct bank quads.
  static constexpr int mrp_calc() {
    int x = ((MR + VW - 1) / VW) * VW;
    if (R == 1) return x;
    while ((x * E) % 32 != 4) x += VW;
    return x;
  }
  static constexpr int MRP = mrp_calc();
  static constexpr int VB = R * MRP;          // elements per vector buffer
  // multi-warp groups publish ahead without a full barrier (see step_arrive)
  // lazy rest-update (see RfKernel::step): one column group per warp only
#ifndef BQR_LAZY
#define BQR_LAZY 1
#endif
  static constexpr bool LAZY = BQR_LAZY != 0 && GT > 32 && R == 32 && !STAGE;
  // Lazy groups are also decoupled: the publishing warp signals a "full"
  // mbarrier per vector buffer and a consumer waits only for that producer
  // (a named barrier with the group's thread count made every step a
  // rendezvous of all warps).  There is no consumer -> producer signal:
  // when v_j is published, every warp w has published its column c in
  // [j-G, j-1] and may still read only v_{c-2} or later, so G + 3 buffers
  // are never overwritten while read.
  static constexpr int NBUF = GT <= 32 ? 2 : (LAZY ? G + 3 : 32 / R + 2);
  static_assert(GT <= 32 || GPB == 1, "multi-warp groups: one group per CTA");
  // [NBUF][VB] vectors | [NMAX] taus | mbarrier (8-byte aligned, 4 words)
  static constexpr int kMbarWord = ((NBUF * VB + NMAX) * E + 3) / 4 * 4;
  static constexpr int kFullWord = kMbarWord + 4;  // LAZY: [NBUF] "full" mbarriers
  static constexpr int kSmallWords = kFullWord + (LAZY ? 2 * NBUF : 0);
  static constexpr int kSmallAll = ((GPB * kSmallWords + 31) / 32) * 32;
  static_assert(R >= 1 && R <= 32 && (R & (R - 1)) == 0, "R must be a power of two <= 32");
  static_assert(GT <= 32 ? (32 % GT == 0) : (GT % 32 == 0 && 32 % R == 0), "group must tile warps");
  static_assert(!STAGE || E == 1, "smem staging implemented for fp32");
  // register rows that may hold the pivot row of a column inside one panel
  static constexpr int NMASK = (G % R == 0) ? G / R : (G + R - 1) / R + 1;
};

template <class T, int R, int G, int MR, int NC, int GPB, bool STAGE, bool EX = false, bool AUG = false>
struct RfKernel {
  using Cfg = RfCfg<T, R, G, MR, NC, GPB, STAGE, EX>;
  using X = El<T>;
  static constexpr int GT = Cfg::GT;
  static constexpr int VW = Cfg::VW;
  static constexpr int MRP = Cfg::MRP;
  static constexpr int VB = Cfg::VB;
  static constexpr int NBUF = Cfg::NBUF;
  static constexpr int MMAX_ = Cfg::MMAX, NMAX_ = Cfg::NMAX;
  // Fully unrolled column loop: ~27% fewer instructions for 56x56, but the
  // ~250 KB of straight-line code thrashes the instruction cache (58% of
  // stall samples "no_inst" on B200), so the panel loop is the default.
  static constexpr bool kFullUnroll = false;
  // 1: one butterfly per column on the owner's chain (apply_look) and the
  // cross-panel look-ahead; correct (parity green) but slower on every
  // measured class (C3 92 -> 140 us, C4 118 -> 130 us: three reflector
  // copies per panel body, profiles/r02/experiments/README.md), so the
  // default is the round-1 chain (dot butterfly, then the norm butterfly)
#ifndef BQR_FUSED_LOOK
#define BQR_FUSED_LOOK 0
#endif
  static constexpr bool kFusedLook = BQR_FUSED_LOOK != 0;
  // the last step of a panel forms the next panel's first reflector
#ifndef BQR_CROSS_PANEL
#define BQR_CROSS_PANEL 1
#endif
  static constexpr bool kCross = BQR_CROSS_PANEL != 0 && kFusedLook;
  static __device__ __forceinline__ int buf(int k) { return k % NBUF; }

  struct Ctx {
    T *vbuf;   // [NBUF][VB]
    T *taus;   // [NMAX]
    int rg, cg, t, lane, grp;
    int wid;   // warp index in the group, warp-uniform by construction (shfl)
    int kmax;
    unsigned long long *full;  // LAZY: [NBUF] full barriers
    int gbase;                 // LAZY: steps published before this matrix
#ifdef BQR_PHASE_TIMING
    bool dbg;
#endif
  };


  struct Look {
    T scal, tau;
    float beta;
  };

  // ------------------------------------------------------------ step signals
  static __device__ __forceinline__ void sig_arrive(Ctx &c, int k) {
    if constexpr (Cfg::LAZY) {
      // every lane of the publishing warp arrives (count 32): each lane's
      // vector stores are released by its own arrive; the warp barrier first
      // orders lane 0's tau store before every lane's arrive (so the release
      // covers it too -- racecheck cannot otherwise prove the tau read of
      // the consumers ordered)
      warp_sync();
      asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(c.full + (c.gbase + k) % NBUF))
                   : "memory");
    } else {
      step_arrive<GT, NBUF>(k);
    }
  }
  static __device__ __forceinline__ void sig_wait(Ctx &c, int k) {
    if constexpr (Cfg::LAZY) {
      const int g = c.gbase + k;
      void *b = c.full + g % NBUF;
      const unsigned par = (unsigned)(g / NBUF) & 1u;
      while (!mbar_try_wait(b, par)) {
      }
    } else {
      step_wait<GT, NBUF>(k);
    }
  }

  // ------------------------------------------------------------ smem vector I/O
  // load rows [I0, MR) of this lane's Householder vector (others left unset)
  template <int I0>
  static __device__ __forceinline__ void load_v(const T *base, T (&v)[MR]) {
#pragma unroll
    for (int q = 0; q < MR; ++q) {
      if (q < I0) continue;
      const int q0 = q - q % VW;
      const bool vec_start = (q % VW == 0) && (q + VW <= MR);
      const bool in_vec = (q % VW != 0) && (q0 >= I0) && (q0 + VW <= MR);
      if (vec_start) {
        const float4 f = lds128(base + q);
        if constexpr (VW == 4) {
          v[q] = X::make(f.x, 0.f);
          v[q + 1 < MR ? q + 1 : q] = X::make(f.y, 0.f);
          v[q + 2 < MR ? q + 2 : q] = X::make(f.z, 0.f);
          v[q + 3 < MR ? q + 3 : q] = X::make(f.w, 0.f);
        } else {
          set_word(v[q], 0, f.x);
          set_word(v[q], 1, f.y);
          set_word(v[q + 1 < MR ? q + 1 : q], 0, f.z);
          set_word(v[q + 1 < MR ? q + 1 : q], 1, f.w);
        }
      } else if (!in_vec) {
        if constexpr (VW == 4) {
          v[q] = X::make(lds32(base + q), 0.f);
        } else {
          const float2 f = lds64(base + q);
          set_word(v[q], 0, f.x);
          set_word(v[q], 1, f.y);
        }
      }
    }
  }

  // ------------------------------------------------------------ reflector
  // xLARFG for column kn held in slot S (rows from register row I0s).
  // Every lane of a warp that contains the owning column group computes it;
  // only the owner's bits are used (Table VI "Column").  Branch-free, so the
  // compiler can interleave it with the independent trailing-update FMAs.
  template <int S, int I0s>
  static __device__ __forceinline__ Look reflector(Ctx &c, const T (&a)[MR][NC], int kn) {
    float s0 = 0.f, s1 = 0.f, s2 = 0.f, s3 = 0.f;
    T alpha = X::zero();
    const int lim = kn - c.rg;  // row r = rg + R i is below the pivot iff R i > lim
#pragma unroll
    for (int i = I0s; i < MR; ++i) {
      const T x = a[i][S];
      T xm = x;
      if (i < I0s + Cfg::NMASK) {
        xm = X::sel(R * i > lim, x, X::zero());
        alpha = X::sel(R * i == lim, x, alpha);
      }
      switch ((i - I0s) & 3) {
        case 0: s0 = X::abs2_acc(xm, s0); break;
        case 1: s1 = X::abs2_acc(xm, s1); break;
        case 2: s2 = X::abs2_acc(xm, s2); break;
        default: s3 = X::abs2_acc(xm, s3); break;
      }
    }
    float sig = (s0 + s1) + (s2 + s3);
    sig = row_allreduce_f<R>(sig);
    if constexpr (R > 1) alpha = X::shfl(alpha, (c.lane & ~(R - 1)) | (kn & (R - 1)));
    const Reflector<T> h = make_reflector(alpha, sig);
    Look l;
    l.scal = h.scal;
    l.tau = h.tau;
    l.beta = h.beta;
    return l;
  }

  // Look-ahead slot P fused with the reflector of column kn = k+1 (the
  // owner's chain of one step, Table VI "Column" after "Trailing Matrix"):
  // H_k is unitary on rows >= k, so the squared norm of the updated column
  // over rows >= k equals gamma = sum_{r >= k} |a_r|^2 of the column BEFORE
  // the update, and nu^2 = |alpha|^2 + sigma = gamma - |a'_k|^2 with a'_k =
  // R_{k,kn} and alpha = a'_kn read from the two updated pivot rows.  gamma
  // rides in the same butterfly as the dot product w = v^H a, so the chain
  // has one row reduction per column instead of two.  The subtraction is
  // accurate while it cancels at most one bit (nu^2 >= gamma / 2); below
  // that, or when sigma may be (near) zero (|alpha|^2 > 15/16 nu^2, e.g. an
  // already triangular column, which must give tau = 0 exactly, reading Q5),
  // the group falls back to the direct masked norm of reflector() -- a
  // warp-uniform branch, rare on dense inputs.
  // S: the slot holding column kn (P, or P + 1 for the cross-panel
  // look-ahead of a panel's last step); rows from I0; register rows
  // [IM, IM + NM) may hold rows k / kn; I0F: first register row of kn's panel
  // (the fallback reflector and its masks).
  template <int S, int I0, int IM, int NM, int I0F>
  static __device__ __forceinline__ Look apply_look(Ctx &c, T (&a)[MR][NC], const T *vb, T ct, int k, bool la) {
    const int kn = k + 1;
    T v[MR];
    load_v<I0>(vb, v);
    T w0 = X::zero(), w1 = X::zero();
    float g0 = 0.f, g1 = 0.f;
    const int limk = k - c.rg;  // row r = rg + R i >= k  <=>  R i >= limk
#pragma unroll
    for (int i = I0; i < MR; ++i) {
      const T x = a[i][S];
      if ((i - I0) & 1) {
        w1 = X::cfma(v[i], x, w1);
      } else {
        w0 = X::cfma(v[i], x, w0);
      }
      const T xm = (i >= IM && i < IM + NM) ? X::sel(R * i >= limk, x, X::zero()) : (i < IM ? X::zero() : x);
      if ((i - I0) & 1) {
        g1 = X::abs2_acc(xm, g1);
      } else {
        g0 = X::abs2_acc(xm, g0);
      }
    }
    T w = X::add(w0, w1);
    float gam = g0 + g1;
    if constexpr (R > 1) {
      if constexpr (X::kComplex) {
        float f[3] = {X::re(w), X::im(w), gam};
#pragma unroll
        for (int o = 1; o < R; o <<= 1) {
#pragma unroll
          for (int q = 0; q < 3; ++q) f[q] += __shfl_xor_sync(0xffffffffu, f[q], o);
        }
        w = X::make(f[0], f[1]);
        gam = f[2];
      } else {
        float f[2] = {X::re(w), gam};
#pragma unroll
        for (int o = 1; o < R; o <<= 1) {
#pragma unroll
          for (int q = 0; q < 2; ++q) f[q] += __shfl_xor_sync(0xffffffffu, f[q], o);
        }
        w = X::make(f[0], 0.f);
        gam = f[1];
      }
    }
    const T t = X::sel(S * G + c.cg > k, X::mul(ct, w), X::zero());
#pragma unroll
    for (int i = I0; i < MR; ++i) a[i][S] = X::fnms(v[i], t, a[i][S]);
    // the updated pivot rows k and kn of this column
    T xk = X::zero(), xa = X::zero();
    const int limn = kn - c.rg;
#pragma unroll
    for (int i = IM; i < MR && i < IM + NM; ++i) {
      xk = X::sel(R * i == limk, a[i][S], xk);
      xa = X::sel(R * i == limn, a[i][S], xa);
    }
    if constexpr (R > 1) {
      xk = X::shfl(xk, (c.lane & ~(R - 1)) | (k & (R - 1)));
      xa = X::shfl(xa, (c.lane & ~(R - 1)) | (kn & (R - 1)));
    }
    const float xk2 = X::abs2_acc(xk, 0.f), xa2 = X::abs2_acc(xa, 0.f);
    const float nu2 = gam - xk2;
    const float sig = nu2 - xa2;
    const bool own = la && ((GT > 32 && R == 32) ? true : (c.cg == kn % G));
    const bool bad = own && !(nu2 >= 0.5f * gam && sig >= 0.0625f * nu2);
    if (__any_sync(0xffffffffu, bad)) return reflector<S, I0F>(c, a, kn);
    const Reflector<T> h = make_reflector(xa, sig);
    Look l;
    l.scal = h.scal;
    l.tau = h.tau;
    l.beta = h.beta;
    return l;
  }

  // Owner lanes (own && on): scale the column, store beta, publish v and
  // tau.  Branch-free, so no divergent region precedes the next shuffles
  // (a divergent branch makes the compiler guard every later shuffle with
  // WARPSYNC): non-owner lanes multiply by 1 (bit-exact no-op) and only the
  // few rows that can hold the pivot need selects.
  template <int S, int I0s>
  static __device__ __forceinline__ void publish(Ctx &c, T (&a)[MR][NC], int kn, const Look &l, bool on) {
    const bool own = on && ((GT > 32 && R == 32) ? true : (c.cg == kn % G));
    const T scal = X::sel(own, l.scal, X::one());
    T *vb = c.vbuf + buf(kn) * VB + c.rg * MRP;
    const int lim = kn - c.rg;
    T v[MR];
#pragma unroll
    for (int i = I0s; i < MR; ++i) {
      const T x = a[i][S];
      const T xs = X::mul(x, scal);
      if (i < I0s + Cfg::NMASK) {
        v[i] = X::sel(R * i > lim, xs, X::sel(R * i == lim, X::one(), X::zero()));
        a[i][S] = X::sel(R * i > lim, xs, X::sel(own && R * i == lim, X::make(l.beta, 0.f), x));
      } else {
        v[i] = xs;
        a[i][S] = xs;
      }
    }
#pragma unroll
    for (int q = I0s; q < MR; ++q) {
      const int q0 = q - q % VW;
      const bool vec_start = (q % VW == 0) && (q + VW <= MR);
      const bool in_vec = (q % VW != 0) && (q0 >= I0s) && (q0 + VW <= MR);
      if (vec_start) {
        float4 f;
        if constexpr (VW == 4) {
          f = make_float4(X::re(v[q]), X::re(v[q + 1 < MR ? q + 1 : q]), X::re(v[q + 2 < MR ? q + 2 : q]),
                          X::re(v[q + 3 < MR ? q + 3 : q]));
        } else {
          const T v1 = v[q + 1 < MR ? q + 1 : q];
          f = make_float4(get_word(v[q], 0), get_word(v[q], 1), get_word(v1, 0), get_word(v1, 1));
        }
        if (own) *reinterpret_cast<float4 *>(vb + q) = f;
      } else if (!in_vec) {
        if (own) vb[q] = v[q];
      }
    }
    if (own && c.rg == 0) c.taus[kn] = l.tau;
  }

  // does this thread's warp hold the column group that owns column kn?
  static __device__ __forceinline__ bool warp_has(const Ctx &c, int kn) {
    if constexpr (GT <= 32) {
      return true;
    } else {
      return ((kn % G) / (32 / R)) == c.wid;
    }
  }
  // can this warp skip slot-P work entirely (all its column groups <= kk)?
  static __device__ __forceinline__ bool warp_done_slot(const Ctx &c, int kk) {
    if constexpr (GT <= 32) {
      return false;
    } else {
      return (c.wid + 1) * (32 / R) - 1 <= kk;
    }
  }

  // ------------------------------------------------------------ packed FP32 (FFMA2)
  // sm_100a issues a packed fp32x2 FMA (fma.rn.f32x2, SASS FFMA2) per lane in
  // one slot: the same IEEE fma on two operand pairs.  The kernels are issue
  // bound (ncu: IPC ~1.9 of 4, FFMA ~53% of the instructions), so the
  // matrix-vector product and the rank-1 update run on row pairs (real) or
  // on the (re, im) pair (complex), halving the FMA issue slots.
#ifndef BQR_FFMA2
#define BQR_FFMA2 1
#endif
  // real tiles: packed across column pairs (BQR_FFMA2_COLS; C3 92.0 -> 90.2 us,
  // f32 128 131.9 -> 127.3 us, profiles/r02/experiments/ab_cols.jsonl)
#ifndef BQR_FFMA2_COLS
#define BQR_FFMA2_COLS 1
#endif
  static constexpr bool kColPairs = BQR_FFMA2_COLS != 0 && !X::kComplex;
  static constexpr bool kPacked = BQR_FFMA2 != 0 && (X::kComplex || MR * NC <= 128 || kColPairs);

  static __device__ __forceinline__ float2 pk(float x, float y) { return make_float2(x, y); }

  // Real: H_k applied to slots [J0, J1) with rows paired (2p, 2p+1); a leading
  // odd row I0 and a trailing odd row MR-1 run as scalar FMAs.  Each product
  // is the same fma as the scalar path; only the summation grouping of the
  // dot products differs (two interleaved partial sums per accumulator).
  template <int P, int I0, int J0, int J1>
  static __device__ __forceinline__ void apply_pk_real(Ctx &c, float (&a)[MR][NC], const float *vb, float ct, int kk,
                                                     bool skip0 = false) {
    constexpr int NS = J1 - J0;
    constexpr int IP = (I0 + 1) & ~1;
    constexpr int NPR = (MR - IP) / 2;
    constexpr bool HEAD = IP > I0 && I0 < MR;
    constexpr bool TAIL = ((MR - IP) & 1) != 0 && IP < MR;
    constexpr int ACC = NS <= 6 ? 2 : 1;
    float2 w2[NS][ACC];
    float ws[NS];
#pragma unroll
    for (int j = 0; j < NS; ++j) {
      ws[j] = 0.f;
#pragma unroll
      for (int q = 0; q < ACC; ++q) w2[j][q] = pk(0.f, 0.f);
    }
    {
      float v[MR];
      load_v<I0>(vb, v);
#pragma unroll
      for (int p = 0; p < NPR; ++p) {
        const int i = IP + 2 * p;
        const float2 v2 = pk(v[i], v[i + 1]);
#pragma unroll
        for (int j = 0; j < NS; ++j)
          w2[j][p % ACC] = __ffma2_rn(v2, pk(a[i][J0 + j], a[i + 1][J0 + j]), w2[j][p % ACC]);
      }
#pragma unroll
      for (int j = 0; j < NS; ++j) {
        if constexpr (HEAD) ws[j] = fmaf(v[I0], a[I0][J0 + j], ws[j]);
        if constexpr (TAIL) ws[j] = fmaf(v[MR - 1], a[MR - 1][J0 + j], ws[j]);
      }
    }
    float sum[NS];
#pragma unroll
    for (int j = 0; j < NS; ++j) {
      float2 s2 = w2[j][0];
      if constexpr (ACC == 2) s2 = __fadd2_rn(s2, w2[j][1]);
      sum[j] = (s2.x + s2.y) + ws[j];
    }
    if constexpr (R >= 8 && NS >= 2) {
      row_allreduce_multi<R, NS>(sum, c.lane);
    } else {
#pragma unroll
      for (int j = 0; j < NS; ++j) sum[j] = row_allreduce<R>(sum[j]);
    }
    float tw[NS];
#pragma unroll
    for (int j = 0; j < NS; ++j) {
      tw[j] = ct * sum[j];
      if (J0 + j == P) tw[j] = c.cg > kk ? tw[j] : 0.f;
      if (j == 0) tw[j] = skip0 ? 0.f : tw[j];
    }
    {
      float v[MR];
      load_v<I0>(vb, v);
#pragma unroll
      for (int j = 0; j < NS; ++j) {
        const float2 nt = pk(-tw[j], -tw[j]);
#pragma unroll
        for (int p = 0; p < NPR; ++p) {
          const int i = IP + 2 * p;
          const float2 r = __ffma2_rn(pk(v[i], v[i + 1]), nt, pk(a[i][J0 + j], a[i + 1][J0 + j]));
          a[i][J0 + j] = r.x;
          a[i + 1][J0 + j] = r.y;
        }
        if constexpr (HEAD) a[I0][J0 + j] = fmaf(-v[I0], tw[j], a[I0][J0 + j]);
        if constexpr (TAIL) a[MR - 1][J0 + j] = fmaf(-v[MR - 1], tw[j], a[MR - 1][J0 + j]);
      }
    }
  }

  // Real, packed across COLUMN pairs (a[i][2q], a[i][2q+1]) at even absolute
  // slot indices (the same pairing in every panel, so the register allocator
  // can keep each pair in an aligned register pair): w_{2q,2q+1} += v_i (a,a'),
  // (a, a') -= v_i (t_{2q}, t_{2q+1}) with v_i as the FFMA2 scalar operand.
  // An odd leading / trailing slot of [J0, J1) runs scalar.
  template <int P, int I0, int J0, int J1>
  static __device__ __forceinline__ void apply_pk_real_cols(Ctx &c, float (&a)[MR][NC], const float *vb, float ct,
                                                            int kk, bool skip0 = false) {
    constexpr int NS = J1 - J0;
    constexpr bool HEADJ = (J0 & 1) != 0;            // slot J0 unpaired
    constexpr int JP = HEADJ ? J0 + 1 : J0;          // first paired slot
    constexpr int NP = (J1 - JP) / 2;                // pairs (JP + 2q, JP + 2q + 1)
    constexpr bool TAILJ = ((J1 - JP) & 1) != 0;     // slot J1 - 1 unpaired
    float2 w2[NP > 0 ? NP : 1];
    float wh = 0.f, wt = 0.f;
#pragma unroll
    for (int q = 0; q < (NP > 0 ? NP : 1); ++q) w2[q] = pk(0.f, 0.f);
    {
      float v[MR];
      load_v<I0>(vb, v);
#pragma unroll
      for (int i = I0; i < MR; ++i) {
#pragma unroll
        for (int q = 0; q < NP; ++q)
          w2[q] = __ffma2_rn(pk(v[i], v[i]), pk(a[i][JP + 2 * q], a[i][JP + 2 * q + 1]), w2[q]);
        if constexpr (HEADJ) wh = fmaf(v[i], a[i][J0], wh);
        if constexpr (TAILJ) wt = fmaf(v[i], a[i][J1 - 1], wt);
      }
    }
    float sum[NS];
    if constexpr (HEADJ) sum[0] = wh;
#pragma unroll
    for (int q = 0; q < NP; ++q) {
      sum[JP - J0 + 2 * q] = w2[q].x;
      sum[JP - J0 + 2 * q + 1] = w2[q].y;
    }
    if constexpr (TAILJ) sum[NS - 1] = wt;
    if constexpr (R >= 8 && NS >= 2) {
      row_allreduce_multi<R, NS>(sum, c.lane);
    } else {
#pragma unroll
      for (int j = 0; j < NS; ++j) sum[j] = row_allreduce<R>(sum[j]);
    }
    float tw[NS];
#pragma unroll
    for (int j = 0; j < NS; ++j) {
      tw[j] = ct * sum[j];
      if (J0 + j == P) tw[j] = c.cg > kk ? tw[j] : 0.f;
      if (j == 0) tw[j] = skip0 ? 0.f : tw[j];
    }
    {
      float v[MR];
      load_v<I0>(vb, v);
#pragma unroll
      for (int q = 0; q < NP; ++q) {
        const float2 nt = pk(-tw[JP - J0 + 2 * q], -tw[JP - J0 + 2 * q + 1]);
#pragma unroll
        for (int i = I0; i < MR; ++i) {
          const float2 r = __ffma2_rn(pk(v[i], v[i]), nt, pk(a[i][JP + 2 * q], a[i][JP + 2 * q + 1]));
          a[i][JP + 2 * q] = r.x;
          a[i][JP + 2 * q + 1] = r.y;
        }
      }
#pragma unroll
      for (int i = I0; i < MR; ++i) {
        if constexpr (HEADJ) a[i][J0] = fmaf(-v[i], tw[0], a[i][J0]);
        if constexpr (TAILJ) a[i][J1 - 1] = fmaf(-v[i], tw[NS - 1], a[i][J1 - 1]);
      }
    }
  }

  // Complex: conj(v) a = (vr, vr) * (ar, ai) + (vi, vi) * (ar, ai) recombined
  // as (A.x + B.y, A.y - B.x); the update a -= v t is
  // a = fma2((vr, vr), (-tr, -ti), a); a = fma2((vi, vi), (ti, -tr), a).
  template <int P, int I0, int J0, int J1>
  static __device__ __forceinline__ void apply_pk_cplx(Ctx &c, float2 (&a)[MR][NC], const float2 *vb, float2 ct,
                                                      int kk, bool skip0 = false) {
    constexpr int NS = J1 - J0;
    float2 wa[NS], wb[NS];
#pragma unroll
    for (int j = 0; j < NS; ++j) wa[j] = wb[j] = pk(0.f, 0.f);
    {
      float2 v[MR];
      load_v<I0>(vb, v);
#pragma unroll
      for (int i = I0; i < MR; ++i) {
        const float2 vr = pk(v[i].x, v[i].x), vi = pk(v[i].y, v[i].y);
#pragma unroll
        for (int j = 0; j < NS; ++j) {
          wa[j] = __ffma2_rn(vr, a[i][J0 + j], wa[j]);
          wb[j] = __ffma2_rn(vi, a[i][J0 + j], wb[j]);
        }
      }
    }
    float f[2 * NS];
#pragma unroll
    for (int j = 0; j < NS; ++j) {
      f[2 * j] = wa[j].x + wb[j].y;
      f[2 * j + 1] = wa[j].y - wb[j].x;
    }
    // (a single slot -- the owner's slot P on the reflector chain -- takes
    // plain butterflies: one dependent shuffle stage fewer than the
    // reduce-scatter + all-gather)
    if constexpr (R >= 8 && NS >= 2) {
      row_allreduce_multi<R, 2 * NS>(f, c.lane);
    } else {
#pragma unroll
      for (int q = 0; q < 2 * NS; ++q) f[q] = row_allreduce_f<R>(f[q]);
    }
    float2 n1[NS], n2[NS];
#pragma unroll
    for (int j = 0; j < NS; ++j) {
      float2 t = X::mul(ct, pk(f[2 * j], f[2 * j + 1]));
      if (J0 + j == P) t = X::sel(c.cg > kk, t, X::zero());
      if (j == 0) t = X::sel(skip0, X::zero(), t);
      n1[j] = pk(-t.x, -t.y);
      n2[j] = pk(t.y, -t.x);
    }
    {
      float2 v[MR];
      load_v<I0>(vb, v);
#pragma unroll
      for (int i = I0; i < MR; ++i) {
        const float2 vr = pk(v[i].x, v[i].x), vi = pk(v[i].y, v[i].y);
#pragma unroll
        for (int j = 0; j < NS; ++j) a[i][J0 + j] = __ffma2_rn(vi, n2[j], __ffma2_rn(vr, n1[j], a[i][J0 + j]));
      }
    }
  }

  template <int P, int I0, int J0, int J1>
  static __device__ __forceinline__ void apply_pk(Ctx &c, T (&a)[MR][NC], const T *vb, T ct, int kk, bool skip0) {
    if constexpr (X::kComplex)
      apply_pk_cplx<P, I0, J0, J1>(c, a, vb, ct, kk, skip0);
    else if constexpr (kColPairs)
      apply_pk_real_cols<P, I0, J0, J1>(c, a, vb, ct, kk, skip0);
    else
      apply_pk_real<P, I0, J0, J1>(c, a, vb, ct, kk, skip0);
  }

  // ------------------------------------------------------------ trailing update
  // Apply H_k^H (vector in vb, conj(tau) = ct) to slots [J0, J1); slot P
  // columns with cg <= kk are excluded (already factored).  The vector is
  // re-read from shared memory in 16-byte chunks for each pass.
  template <int P, int I0, int J0, int J1>
  // skip0: leave slot J0 alone (the cross-panel look-ahead already applied
  // H_k to it); a uniform select on its multiplier
  static __device__ __forceinline__ void apply(Ctx &c, T (&a)[MR][NC], const T *vb, T ct, int kk, bool skip0 = false) {
    if constexpr (kPacked && J0 < J1) {
      apply_pk<P, I0, J0, J1>(c, a, vb, ct, kk, skip0);
    } else if constexpr (J0 < J1) {
      constexpr int NS = J1 - J0;
      // partial sums per slot: ptxas walks the slots one after another, so a
      // single accumulator per slot is a 4-cycle-per-row serial chain; 4 is
      // best when few slots are live (measured on C3/C4), fewer with many
      // slots to bound the accumulator registers (NS x ACC)
      constexpr int ACC = NS <= 6 ? 4 : (NS <= 12 ? 2 : 1);
      T w[NS][ACC];
#pragma unroll
      for (int j = 0; j < NS; ++j)
#pragma unroll
        for (int q = 0; q < ACC; ++q) w[j][q] = X::zero();
      {
        T v[MR];
        load_v<I0>(vb, v);
#pragma unroll
        for (int i = I0; i < MR; ++i)
#pragma unroll
          for (int j = 0; j < NS; ++j) w[j][(i - I0) % ACC] = X::cfma(v[i], a[i][J0 + j], w[j][(i - I0) % ACC]);
      }
      T tw[NS];
      T sum[NS];
#pragma unroll
      for (int j = 0; j < NS; ++j) {
        T s = w[j][0];
#pragma unroll
        for (int q = 1; q < ACC; ++q) s = X::add(s, w[j][q]);
        sum[j] = s;
      }
      if constexpr (R >= 8 && NS * Cfg::E >= 2 && NS >= 2) {
        // several values over >= 8 row lanes: reduce-scatter + all-gather
        float f[NS * Cfg::E];
#pragma unroll
        for (int j = 0; j < NS; ++j)
#pragma unroll
          for (int e = 0; e < Cfg::E; ++e) f[j * Cfg::E + e] = get_word(sum[j], e);
        row_allreduce_multi<R, NS * Cfg::E>(f, c.lane);
#pragma unroll
        for (int j = 0; j < NS; ++j)
#pragma unroll
          for (int e = 0; e < Cfg::E; ++e) set_word(sum[j], e, f[j * Cfg::E + e]);
      } else {
#pragma unroll
        for (int j = 0; j < NS; ++j) sum[j] = row_allreduce<R>(sum[j]);
      }
#pragma unroll
      for (int j = 0; j < NS; ++j) {
        tw[j] = X::mul(ct, sum[j]);
        if (J0 + j == P) tw[j] = X::sel(c.cg > kk, tw[j], X::zero());
        if (j == 0) tw[j] = X::sel(skip0, X::zero(), tw[j]);
      }
      {
        T v[MR];
        load_v<I0>(vb, v);
#pragma unroll
        for (int i = I0; i < MR; ++i)
#pragma unroll
          for (int j = 0; j < NS; ++j) a[i][J0 + j] = X::fnms(v[i], tw[j], a[i][J0 + j]);
      }
    }
  }

  // panel prologue: reflector for the panel's first column (no look-ahead
  // across panels, which keeps one step body per panel)
  template <int P, int I0>
  static __device__ __forceinline__ void panel_head(Ctx &c, T (&a)[MR][NC], int k) {
    if (warp_has(c, k)) {
      const Look l = reflector<P, I0>(c, a, k);
      publish<P, I0>(c, a, k, l, true);
      sig_arrive(c, k);
    }
  }

  // one Householder step on column k of panel P (first live register row I0):
  // apply H_k to slot P, form + publish reflector k+1 (same slot), then apply
  // H_k to the remaining slots while the reflector chain drains.  The last
  // step of a panel (kCross) runs the look-ahead on slot P + 1 instead --
  // column k+1 opens the next panel -- so no panel starts with a reflector
  // that nothing overlaps (panel_head runs for panel 0 only).
  template <int P, int I0>
  static __device__ __forceinline__ Look look(Ctx &c, T (&a)[MR][NC], const T *vb, T ct, int k, bool la) {
    if constexpr (kFusedLook) {
      return apply_look<P, I0, I0, Cfg::NMASK, I0>(c, a, vb, ct, k, la);
    } else {
      apply<P, I0, P, P + 1>(c, a, vb, ct, k - P * G);
      return reflector<P, I0>(c, a, k + 1);
    }
  }
  // look-ahead across the panel boundary: H_k on slot P + 1 and reflector
  // k+1 = (P+1) G from it (rows from I0; the pivot rows k, k+1 lie in
  // register rows [I0, I0 + NMASK + 1); the next panel starts at row I0N)
  template <int P, int I0>
  static __device__ __forceinline__ Look look_x(Ctx &c, T (&a)[MR][NC], const T *vb, T ct, int k, bool la) {
    constexpr int PN = P + 1 < NC ? P + 1 : P;
    constexpr int I0N = (PN * G) / R;
    return apply_look<PN, I0, I0, Cfg::NMASK + 1, I0N>(c, a, vb, ct, k, la);
  }
  template <int P>
  static __device__ __forceinline__ void publish_x(Ctx &c, T (&a)[MR][NC], int kn, const Look &l, bool on) {
    constexpr int PN = P + 1 < NC ? P + 1 : P;
    constexpr int I0N = (PN * G) / R;
    publish<PN, I0N>(c, a, kn, l, on);
  }

  template <int P, int I0>
  static __device__ __forceinline__ void step(Ctx &c, T (&a)[MR][NC], int k) {
    const int kk = k - P * G;
    BQR_STAMP(c, k, 0);
    if (!warp_has(c, k) || GT <= 32) sig_wait(c, k);
    BQR_STAMP(c, k, 1);
    const T ct = X::conj(c.taus[k]);
    const T *vb = c.vbuf + buf(k) * VB + c.rg * MRP;
    const bool la = kk + 1 < G && k + 1 < c.kmax && warp_has(c, k + 1);
    // cross-panel look-ahead (last step of the panel, a next panel exists)
    const bool lastx = kCross && (P + 1 < NC) && kk == G - 1 && k + 1 < c.kmax;
    const bool lax = lastx && warp_has(c, k + 1);
    if constexpr (Cfg::LAZY) {
      // CTA groups, one column group per warp (decoupled signalling).
      // Only the owners of columns k+1 and k+2 need slot P first: the owner
      // of k+1 forms reflector k+1 from it (look-ahead) and publishes before
      // anything else; the owner of k+2 applies H_k to slot P only and
      // defers its other slots to step k+1, after it has published v_{k+2}
      // (lazy rest-update: otherwise that rest-update sits between v_{k+1}
      // arriving and the chain of column k+2).  Every other warp applies
      // H_k to all its live slots in one pass: one reduce-scatter instead
      // of a separate slot-P butterfly.
      const bool defer = kk + 2 < G && k + 2 < c.kmax && warp_has(c, k + 2);
      const bool done = warp_done_slot(c, kk);
      int npass;  // rest-updates H_q (slots P+1..), q = k - npass + 1 .. k
      bool skip = false;
      if (la || defer) {
        if (la) {
          const Look l = look<P, I0>(c, a, vb, ct, k, true);
          publish<P, I0>(c, a, k + 1, l, true);
          sig_arrive(c, k + 1);
          BQR_STAMP(c, k, 2);
        } else {
          apply<P, I0, P, P + 1>(c, a, vb, ct, kk);
        }
        npass = la ? (kk >= 1 ? 2 : 1) : 0;  // + the rest deferred at step k-1
      } else if (lax) {
        const Look l = look_x<P, I0>(c, a, vb, ct, k, true);
        publish_x<P>(c, a, k + 1, l, true);
        sig_arrive(c, k + 1);
        npass = 1;
        skip = true;
      } else if (done) {
        npass = 1;
      } else {
        apply<P, I0, P, NC>(c, a, vb, ct, kk);
        npass = 0;
      }
      // one call site for every rest-update (the apply body is inlined per
      // call site; fewer copies keep the panel code in the instruction cache)
#pragma unroll 1
      for (int q = k - npass + 1; q <= k; ++q)
        apply<P, I0, P + 1, NC>(c, a, c.vbuf + buf(q) * VB + c.rg * MRP, X::conj(c.taus[q]), q - P * G,
                                skip && q == k);
      BQR_STAMP(c, k, 3);
      return;
    }
    if constexpr (GT <= 32) {
      // sub-warp groups: the reflector chain (computed unconditionally, no
      // branch around its shuffles) overlaps the remaining updates in one
      // basic block; the owner lanes publish at the end of the step
      // (one call site of the rest-update; the second test of lastx is
      // opaque so the compiler does not thread the branch through it by
      // duplicating the update)
      Look l;
      if (lastx) {
        l = look_x<P, I0>(c, a, vb, ct, k, true);
      } else {
        l = look<P, I0>(c, a, vb, ct, k, la);
      }
      apply<P, I0, P + 1, NC>(c, a, vb, ct, kk, lastx);
      if (opaque(lastx ? 1 : 0)) {
        publish_x<P>(c, a, k + 1, l, true);
      } else {
        publish<P, I0>(c, a, k + 1, l, la);
      }
      BQR_STAMP(c, k, 3);
    } else {
      // multi-warp groups: publish first so the other warps never wait
      bool skip = false;
      if (la) {
        const Look l = look<P, I0>(c, a, vb, ct, k, true);
        publish<P, I0>(c, a, k + 1, l, true);
        sig_arrive(c, k + 1);
      } else if (lax) {
        const Look l = look_x<P, I0>(c, a, vb, ct, k, true);
        publish_x<P>(c, a, k + 1, l, true);
        sig_arrive(c, k + 1);
        skip = true;
      } else if (!warp_done_slot(c, kk)) {
        apply<P, I0, P, P + 1>(c, a, vb, ct, kk);
      }
      BQR_STAMP(c, k, 2);
      apply<P, I0, P + 1, NC>(c, a, vb, ct, kk, skip);
      BQR_STAMP(c, k, 3);
    }
  }

  // ====================================================================
  // Fully unrolled variant (UNR): the column index is a compile-time
  // constant after unrolling, so row ranges are exact (no panel waste) and
  // almost every pivot mask folds away; only the lane-dependent row offset
  // rg and the slot-mask cg > kk remain runtime.  Used for sub-warp groups of
  // exact-shape classes (e.g. 2 x 56x56 fp32 per warp), where the masks and
  // panel waste were ~30% of all issued instructions.
  // ====================================================================
  // r = rg + R i vs the pivot kn (folds to a constant unless i straddles kn)
  static __device__ __forceinline__ bool row_gt(const Ctx &c, int i, int kn) {
    return (R * i > kn) ? true : ((R * i + R - 1 <= kn) ? false : (R * i > kn - c.rg));
  }
  static __device__ __forceinline__ bool row_eq(const Ctx &c, int i, int kn) {
    return (R * i > kn || R * i + R - 1 < kn) ? false : (R * i == kn - c.rg);
  }

  static __device__ __forceinline__ Look ureflector(Ctx &c, const T (&a)[MR][NC], int kn, int S) {
    float s0 = 0.f, s1 = 0.f, s2 = 0.f, s3 = 0.f;
    T alpha = X::zero();
    const int i0 = kn / R;
#pragma unroll
    for (int i = 0; i < MR; ++i) {
      if (i < i0) continue;
      const T x = a[i][S];
      const T xm = X::sel(row_gt(c, i, kn), x, X::zero());
      alpha = X::sel(row_eq(c, i, kn), x, alpha);
      switch ((i - i0) & 3) {
        case 0: s0 = X::abs2_acc(xm, s0); break;
        case 1: s1 = X::abs2_acc(xm, s1); break;
        case 2: s2 = X::abs2_acc(xm, s2); break;
        default: s3 = X::abs2_acc(xm, s3); break;
      }
    }
    float sig = (s0 + s1) + (s2 + s3);
    sig = row_allreduce_f<R>(sig);
    if constexpr (R > 1) alpha = X::shfl(alpha, (c.lane & ~(R - 1)) | (kn & (R - 1)));
    const Reflector<T> h = make_reflector(alpha, sig);
    Look l;
    l.scal = h.scal;
    l.tau = h.tau;
    l.beta = h.beta;
    return l;
  }

  static __device__ __forceinline__ void upublish(Ctx &c, T (&a)[MR][NC], int kn, int S, const Look &l) {
    const bool own = c.cg == kn % G;
    const T scal = X::sel(own, l.scal, X::one());
    T *vb = c.vbuf + buf(kn) * VB + c.rg * MRP;
    const int i0 = kn / R;
#pragma unroll
    for (int i = 0; i < MR; ++i) {
      if (i < i0) continue;
      const T x = a[i][S];
      const T xs = X::mul(x, scal);
      const bool gt = row_gt(c, i, kn), eq = row_eq(c, i, kn);
      const T v = X::sel(gt, xs, X::sel(eq, X::one(), X::zero()));
      a[i][S] = X::sel(gt, xs, X::sel(own && eq, X::make(l.beta, 0.f), x));
      if (own) vb[i] = v;
    }
    if (own && c.rg == 0) c.taus[kn] = l.tau;
  }

  // H_k^H applied to slots [J0, J1) over register rows [i0, MR)
  static __device__ __forceinline__ void uapply(Ctx &c, T (&a)[MR][NC], const T *vb, T ct, int k, int J0, int J1) {
    const int P = k / G, kk = k % G, i0 = k / R;
    const int NS = J1 - J0;
    if (NS <= 0) return;
    const int ACC = NS >= 4 ? 1 : (NS >= 2 ? 2 : 4);
    T w[NC][4];
#pragma unroll
    for (int j = 0; j < NC; ++j)
#pragma unroll
      for (int q = 0; q < 4; ++q) w[j][q] = X::zero();
#pragma unroll
    for (int i = 0; i < MR; ++i) {
      if (i < i0) continue;
      const T v = vb[i];
#pragma unroll
      for (int j = 0; j < NC; ++j) {
        if (j < J0 || j >= J1) continue;
        w[j][(i - i0) % ACC] = X::cfma(v, a[i][j], w[j][(i - i0) % ACC]);
      }
    }
    T tw[NC];
#pragma unroll
    for (int j = 0; j < NC; ++j) {
      if (j < J0 || j >= J1) continue;
      T s = w[j][0];
#pragma unroll
      for (int q = 1; q < 4; ++q)
        if (q < ACC) s = X::add(s, w[j][q]);
      s = row_allreduce<R>(s);
      tw[j] = X::mul(ct, s);
      if (j == P) tw[j] = X::sel(c.cg > kk, tw[j], X::zero());
    }
    asm volatile("" ::: "memory");  // re-read v for the update (keeps it out of registers)
#pragma unroll
    for (int i = 0; i < MR; ++i) {
      if (i < i0) continue;
      const T v = vb[i];
#pragma unroll
      for (int j = 0; j < NC; ++j) {
        if (j < J0 || j >= J1) continue;
        a[i][j] = X::fnms(v, tw[j], a[i][j]);
      }
    }
  }

  template <int K>
  static __device__ __forceinline__ void ustep(Ctx &c, T (&a)[MR][NC], int kmax) {
    constexpr int P = K / G, kk = K % G;
    constexpr int lo = (kk == G - 1) ? P + 1 : P;
    step_wait<GT, NBUF>(K);
    const T ct = X::conj(c.taus[K]);
    const T *vb = c.vbuf + buf(K) * VB + c.rg * MRP;
    // live slots [lo, NC); slot lo holds column K+1: H_K on it first, then
    // reflector K+1 (unconditional: no branch around its shuffles), then the
    // remaining slots while the reflector chain drains, then the owner lanes
    // publish v_{K+1}
    if constexpr (lo < NC) {
      uapply(c, a, vb, ct, K, lo, lo + 1);
      const Look l = ureflector(c, a, K + 1, lo);
      uapply(c, a, vb, ct, K, lo + 1, NC);
      if (K + 1 < kmax) upublish(c, a, K + 1, lo, l);
    }
  }

  template <int K>
  static __device__ __forceinline__ void usteps(Ctx &c, T (&a)[MR][NC], int kmax) {
    if constexpr (K < NMAX_ && K < MMAX_) {
      if (EX || K < kmax) {
        ustep<K>(c, a, kmax);
        usteps<K + 1>(c, a, kmax);
      }
    }
  }

  static __device__ __forceinline__ void ufactor(Ctx &c, T (&a)[MR][NC]) {
    const int kmax = EX ? (MMAX_ < NMAX_ ? MMAX_ : NMAX_) : c.kmax;
    {
      const Look l = ureflector(c, a, 0, 0);
      if (kmax > 0) upublish(c, a, 0, 0, l);
    }
    usteps<0>(c, a, kmax);
  }

  struct NoHook {
    __device__ __forceinline__ void operator()() const {}
  };

  // panel recursion; `hook` runs once, before panel 1 (or at the end when
  // there is a single panel) -- the persistent warp loop issues its deferred
  // prefetch there, once the previous bulk store has surely read the tile
  template <int P, class H = NoHook>
  static __device__ __forceinline__ void panels(Ctx &c, T (&a)[MR][NC], const H &hook = H()) {
    if constexpr (P < NC) {
      if constexpr (P == 1) hook();
      constexpr int I0 = (P * G) / R;
      const int kbeg = P * G;
      if (kbeg >= c.kmax) {
        if constexpr (P == 0) hook();
        return;
      }
      const int kend = min(kbeg + G, c.kmax);
      if (P == 0 || !kCross) panel_head<P, I0>(c, a, kbeg);
#pragma unroll 1
      for (int k = kbeg; k < kend; ++k) step<P, I0>(c, a, k);
      panels<P + 1>(c, a, hook);
      if constexpr (P == 0 && NC == 1) hook();
    }
  }

  // ---- xORG2R / xUNG2R: Q = H_0 ... H_{k-1} applied backwards (i = k-1 .. 0)
  template <int P, int I0>
  static __device__ __forceinline__ void org_column(Ctx &c, T (&a)[MR][NC], int i, const T *tau_g) {
    const int kk = i - P * G;
    T *vb = c.vbuf + buf(i) * VB + c.rg * MRP;
    const T ti = tau_g[i];
    if (c.cg == kk) {
#pragma unroll
      for (int ii = I0; ii < MR; ++ii) {
        const int r = c.rg + R * ii;
        vb[ii] = X::sel(r > i, a[ii][P], X::sel(r == i, X::one(), X::zero()));
      }
    }
    group_sync<GT, GPB>(c.grp);
    T v[MR];
#pragma unroll
    for (int ii = I0; ii < MR; ++ii) v[ii] = vb[ii];
    T tw[NC];
#pragma unroll
    for (int j = P; j < NC; ++j) {
      T w = X::zero();
#pragma unroll
      for (int ii = I0; ii < MR; ++ii) w = X::cfma(v[ii], a[ii][j], w);
      w = row_allreduce<R>(w);
      tw[j] = X::mul(ti, w);
      if (j == P) tw[j] = X::sel(c.cg > kk, tw[j], X::zero());
    }
#pragma unroll
    for (int j = P; j < NC; ++j) {
#pragma unroll
      for (int ii = I0; ii < MR; ++ii) a[ii][j] = X::fnms(v[ii], tw[j], a[ii][j]);
    }
    if (c.cg == kk) {
      const T mt = X::neg(ti);
      const T d = X::sub(X::one(), ti);
#pragma unroll
      for (int ii = 0; ii < MR; ++ii) {
        const int r = c.rg + R * ii;
        if (ii < I0) {
          a[ii][P] = X::zero();
        } else {
          a[ii][P] = X::sel(r > i, X::mul(mt, v[ii]), X::sel(r == i, d, X::zero()));
        }
      }
    }
  }

  template <int P>
  static __device__ __forceinline__ void org_panels(Ctx &c, T (&a)[MR][NC], int kref, const T *tau_g) {
    if constexpr (P >= 0) {
      constexpr int I0 = (P * G) / R;
      const int kbeg = P * G;
      if (kbeg < kref) {
        const int kend = min(kbeg + G, kref);
#pragma unroll 1
        for (int i = kend - 1; i >= kbeg; --i) org_column<P, I0>(c, a, i, tau_g);
      }
      org_panels<P - 1>(c, a, kref, tau_g);
    }
  }

  // ------------------------------------------------------------ staging
  // in-bounds test; compile-time true for exact-shape instantiations
  static __device__ __forceinline__ bool inb(int r, int col, int m, int n) {
    if constexpr (EX) return true;
    return r < m && col < n;
  }

  // mat: this group's matrix index (the right-hand sides of the augmented
  // classes live at p.B + mat * strideB)
  static __device__ __forceinline__ void load_matrix(const RfArgs &p, Ctx &c, float *smem, T *Ab, long long mat,
                                                     bool active,
                                                     T (&a)[MR][NC]) {
    const int m = p.m, n = p.n;
    if constexpr (STAGE) {
      float *tile = smem + Cfg::kSmallAll + c.grp * p.tileWords;
      const float *Ag = reinterpret_cast<const float *>(Ab);
      if (p.bulk) {
        // one TMA bulk copy of the whole (contiguous) matrix
        void *bar = smem + c.grp * Cfg::kSmallWords + Cfg::kMbarWord;
        if (c.t == 0) mbar_init(bar, 1);
        group_sync<GT, GPB>(c.grp);
        if (c.t == 0 && active) bulk_load(tile, Ag, (unsigned)(m * n * 4), bar);
        // every lane waits on the barriers of ALL groups sharing its warp, so
        // the warp leaves the loop converged (per-group exits would leave the
        // two matrices of a warp running diverged for the whole kernel)
        constexpr int GPW = GT <= 32 ? 32 / GT : 1;
        const int g0 = GT <= 32 ? (c.grp / GPW) * GPW : c.grp;
        bool done = false;
        while (!done) {
          done = true;
#pragma unroll
          for (int g = 0; g < GPW; ++g) {
            void *bg = smem + (g0 + g) * Cfg::kSmallWords + Cfg::kMbarWord;
            const long long mg = (long long)blockIdx.x * GPB + g0 + g;
            if (mg < p.batch) done = mbar_try_wait(bg, 0) && done;
          }
        }
      } else if (active) {
        if (p.vec4 && p.lda == p.ldS) {
          const int nch = (m * n) >> 2;  // contiguous matrix: linear 16-byte copy
          for (int q = c.t; q < nch; q += GT) cp_async16(tile + 4 * q, Ag + 4 * q);
          cp_async_wait_all();
        } else if (p.vec4) {
          const int mq = m >> 2;
          for (int col = 0; col < n; ++col)
            for (int q = c.t; q < mq; q += GT) cp_async16(tile + 4 * q + col * p.ldS, Ag + 4 * q + (long long)col * p.lda);
          cp_async_wait_all();
        } else {
          for (int col = 0; col < n; ++col)
            for (int q = c.t; q < m; q += GT) tile[q + col * p.ldS] = Ag[q + (long long)col * p.lda];
        }
      }
      group_sync<GT, GPB>(c.grp);
      const int ld = EX ? R * MR : p.ldS;
#pragma unroll
      for (int i = 0; i < MR; ++i)
#pragma unroll
        for (int j = 0; j < NC; ++j) {
          const int r = c.rg + R * i, col = c.cg + G * j;
          a[i][j] = (inb(r, col, m, n) && (EX || active)) ? tile[r + col * ld] : 0.f;
        }
    } else {
      const T *Bb = reinterpret_cast<const T *>(p.B) + mat * p.strideB;
#pragma unroll
      for (int i = 0; i < MR; ++i)
#pragma unroll
        for (int j = 0; j < NC; ++j) {
          const int r = c.rg + R * i, col = c.cg + G * j;
          T x = X::zero();
          if (active && inb(r, col, m, n)) x = Ab[r + (long long)col * p.lda];
          if (AUG && active && r < m && col >= n && col < n + p.nrhs) x = Bb[r + (long long)(col - n) * p.ldb];
          a[i][j] = x;
        }
    }
  }

  static __device__ __forceinline__ int opaque(int x) {
    asm volatile("mov.b32 %0, %0;" : "+r"(x));
    return x;
  }

  static __device__ __forceinline__ void store_matrix(const RfArgs &p, Ctx &c, float *smem, T *Ab, long long mat,
                                                      bool active,
                                                      const T (&a)[MR][NC]) {
    // opaque reads: keeps ptxas from hoisting the store's per-element
    // predicates above the factorisation loop (they would stay live in
    // registers through it)
    const int m = opaque(p.m), n = opaque(p.n);
    if constexpr (STAGE) {
      float *tile = smem + Cfg::kSmallAll + c.grp * p.tileWords;
      float *Ag = reinterpret_cast<float *>(Ab);
      const int ld = EX ? R * MR : p.ldS;
      group_sync<GT, GPB>(c.grp);
#pragma unroll
      for (int i = 0; i < MR; ++i)
#pragma unroll
        for (int j = 0; j < NC; ++j) {
          const int r = c.rg + R * i, col = c.cg + G * j;
          if (inb(r, col, m, n)) tile[r + col * ld] = a[i][j];
        }
      // opaque copy of the flag: keeps the compiler from duplicating the whole
      // factorisation to thread the load-time branch into the store
      int bulk;
      asm volatile("mov.b32 %0, %1;" : "=r"(bulk) : "r"(p.bulk));
      if (bulk) {
        fence_async_smem();
        group_sync<GT, GPB>(c.grp);
        if (c.t == 0 && active) {
          bulk_store(Ag, tile, (unsigned)(m * n * 4));
          bulk_store_drain();
        }
        return;
      }
      group_sync<GT, GPB>(c.grp);
      if (active) {
        if (p.vec4 && p.lda == p.ldS) {
          const int nch = (m * n) >> 2;
          for (int q = c.t; q < nch; q += GT)
            *reinterpret_cast<float4 *>(Ag + 4 * q) = *reinterpret_cast<const float4 *>(tile + 4 * q);
        } else if (p.vec4) {
          const int mq = m >> 2;
          for (int col = 0; col < n; ++col)
            for (int q = c.t; q < mq; q += GT)
              *reinterpret_cast<float4 *>(Ag + 4 * q + (long long)col * p.lda) =
                  *reinterpret_cast<const float4 *>(tile + 4 * q + col * p.ldS);
        } else {
          for (int col = 0; col < n; ++col)
            for (int q = c.t; q < m; q += GT) Ag[q + (long long)col * p.lda] = tile[q + col * p.ldS];
        }
      }
    } else if (active) {
      T *Bb = reinterpret_cast<T *>(p.B) + mat * p.strideB;
#pragma unroll
      for (int i = 0; i < MR; ++i)
#pragma unroll
        for (int j = 0; j < NC; ++j) {
          const int r = c.rg + R * i, col = c.cg + G * j;
          if (inb(r, col, m, n)) Ab[r + (long long)col * p.lda] = a[i][j];
          if (AUG && r < m && col >= n && col < n + p.nrhs) Bb[r + (long long)(col - n) * p.ldb] = a[i][j];
        }
    }
  }

  // ====================================================================
  // Persistent CTA loop (multi-warp groups, direct staging): the CTA walks
  // matrices blockIdx.x, +gridDim.x, ...; while it factors one, a TMA bulk
  // copy prefetches the next contiguous matrix into shared memory, so only
  // the first load per CTA is exposed (STAP: 256 matrices on 148 SMs, the
  // second matrix of an SM used to wait ~µs for HBM with the SM idle).
  // ====================================================================
  static __device__ __forceinline__ void run_cta_loop(const RfArgs &p) {
    extern __shared__ __align__(16) float smem[];
    const int t = threadIdx.x;
    Ctx c;
    c.t = t;
    c.grp = 0;
    c.rg = t % R;
    c.cg = t / R;
    c.lane = t & 31;
    c.wid = __shfl_sync(0xffffffffu, t >> 5, 0);
    c.kmax = p.kmax;
#ifdef BQR_PHASE_TIMING
    c.dbg = blockIdx.x == 0;
#endif
    c.vbuf = reinterpret_cast<T *>(smem);
    c.taus = c.vbuf + NBUF * VB;
    T *tile = reinterpret_cast<T *>(smem + Cfg::kSmallAll);
    void *bar = smem + Cfg::kMbarWord;
    const int m = p.m, n = p.n;
    c.full = reinterpret_cast<unsigned long long *>(smem + Cfg::kFullWord);
    c.gbase = 0;
    if (p.bulk || Cfg::LAZY) {
      if (t == 0) {
        if (p.bulk) mbar_init(bar, 1);
        if constexpr (Cfg::LAZY)
          for (int b = 0; b < NBUF; ++b) mbar_init(c.full + b, 32);
      }
      __syncthreads();
    }
    bool have_tile = false;
    unsigned phase = 0;
#pragma unroll 1
    for (long long mat = blockIdx.x; mat < p.batch; mat += gridDim.x) {
      T *Ab = reinterpret_cast<T *>(p.A) + mat * p.strideA;
      T a[MR][NC];
      if (have_tile) {
        while (!mbar_try_wait(bar, phase)) {
        }
        phase ^= 1;
#pragma unroll
        for (int i = 0; i < MR; ++i)
#pragma unroll
          for (int j = 0; j < NC; ++j) {
            const int r = c.rg + R * i, col = c.cg + G * j;
            a[i][j] = inb(r, col, m, n) ? tile[r + col * m] : X::zero();
          }
        if constexpr (AUG) {
          const T *Bb = reinterpret_cast<const T *>(p.B) + mat * p.strideB;
#pragma unroll
          for (int i = 0; i < MR; ++i)
#pragma unroll
            for (int j = 0; j < NC; ++j) {
              const int r = c.rg + R * i, col = c.cg + G * j;
              if (r < m && col >= n && col < n + p.nrhs) a[i][j] = Bb[r + (long long)(col - n) * p.ldb];
            }
        }
      } else {
        load_matrix(p, c, smem, Ab, mat, true, a);
      }
      __syncthreads();  // tile consumed by every thread
      const long long nxt = mat + gridDim.x;
      have_tile = p.bulk && nxt < p.batch;
      if (have_tile && t == 0) {
        fence_async_smem();
        bulk_load(tile, reinterpret_cast<const T *>(p.A) + nxt * p.strideA, (unsigned)(m * n * sizeof(T)), bar);
      }
      panels<0>(c, a);
#ifdef BQR_PHASE_TIMING
      c.dbg = false;
#endif
      __syncthreads();  // every tau published before the tau store
      store_matrix(p, c, smem, Ab, mat, true, a);
      T *tg = reinterpret_cast<T *>(p.tau) + mat * p.strideT;
      for (int idx = t; idx < p.kmax; idx += GT) tg[idx] = c.taus[idx];
      __syncthreads();  // vector/tau buffers reused by the next matrix
      c.gbase += p.kmax;
    }
  }

  // ====================================================================
  // Persistent warp loop (sub-warp groups, exact contiguous shapes): each
  // warp walks matrix groups blockIdx.x, +gridDim.x, ...  The group's
  // shared-memory tile always holds the NEXT input (TMA bulk prefetch, issued
  // while the current matrix is factored); at the end of a matrix every lane
  // swaps its result elements with the next input's elements at the same
  // positions (so the tile becomes the output, the registers the next input),
  // a bulk store drains the tile, and the prefetch after that is deferred to
  // panel 1 of the next factorisation.  Loads and stores overlap compute
  // except for the very first load and last store of a warp.
  // ====================================================================
  static __device__ __forceinline__ void run_warp_loop(const RfArgs &p) {
    extern __shared__ __align__(16) float smem[];
    const int tid = threadIdx.x;
    const int grp = tid / GT;
    const int t = tid - grp * GT;
    Ctx c;
    c.t = t;
    c.grp = grp;
    c.rg = t % R;
    c.cg = t / R;
    c.lane = tid & 31;
    c.wid = 0;
    c.kmax = MMAX_ < NMAX_ ? MMAX_ : NMAX_;
#ifdef BQR_PHASE_TIMING
    c.dbg = blockIdx.x == 0;
#endif
    c.vbuf = reinterpret_cast<T *>(smem + grp * Cfg::kSmallWords);
    c.taus = c.vbuf + NBUF * VB;
    float *tile = smem + Cfg::kSmallAll + grp * p.tileWords;
    void *bar = smem + grp * Cfg::kSmallWords + Cfg::kMbarWord;
    constexpr int LD = MMAX_;
    constexpr unsigned kBytes = MMAX_ * NMAX_ * 4;
    const long long nitems = (p.batch + GPB - 1) / GPB;
    auto matof = [&](long long q) { return q * GPB + grp; };
    auto gptr = [&](long long mat) { return reinterpret_cast<float *>(p.A) + mat * p.strideA; };
    if (t == 0) mbar_init(bar, 1);
    warp_sync();
    long long q = blockIdx.x;
    if (q >= nitems) return;
    // every lane waits on ALL groups' barriers of its warp: converged exit
    auto wait_tiles = [&](unsigned phase, long long item) {
      bool done = false;
      while (!done) {
        done = true;
#pragma unroll
        for (int g = 0; g < GPB; ++g) {
          void *bg = smem + g * Cfg::kSmallWords + Cfg::kMbarWord;
          if (item * GPB + g < p.batch) done = mbar_try_wait(bg, phase) && done;
        }
      }
    };
    unsigned phase = 0;
    if (t == 0 && matof(q) < p.batch) bulk_load(tile, gptr(matof(q)), kBytes, bar);
    wait_tiles(phase, q);
    phase ^= 1;
    T a[MR][NC];
#pragma unroll
    for (int i = 0; i < MR; ++i)
#pragma unroll
      for (int j = 0; j < NC; ++j) a[i][j] = tile[(c.rg + R * i) + (c.cg + G * j) * LD];
    warp_sync();
    long long pending = q + gridDim.x;  // prefetch target, issued at the hook
    if (pending < nitems) {
      if (t == 0 && matof(pending) < p.batch) bulk_load(tile, gptr(matof(pending)), kBytes, bar);
      pending = -1;
    }
#pragma unroll 1
    for (; q < nitems; q += gridDim.x) {
      const long long mat = matof(q);
      const bool valid = mat < p.batch;
      auto hook = [&]() {
        if (pending >= 0) {
          if (t == 0) {
            bulk_store_drain();  // the previous output left the tile
            if (matof(pending) < p.batch) bulk_load(tile, gptr(matof(pending)), kBytes, bar);
          }
          pending = -1;
        }
      };
      panels<0>(c, a, hook);
#ifdef BQR_PHASE_TIMING
      c.dbg = false;
#endif
      warp_sync();
      const long long qn = q + gridDim.x;
      if (qn < nitems) {
        wait_tiles(phase, qn);
        phase ^= 1;
#pragma unroll
        for (int i = 0; i < MR; ++i)
#pragma unroll
          for (int j = 0; j < NC; ++j) {
            float *e = tile + (c.rg + R * i) + (c.cg + G * j) * LD;
            const float x = *e;
            *e = a[i][j];
            a[i][j] = x;
          }
      } else {
        // last matrix of this warp: the previous iteration's bulk store may
        // still be reading the tile when no prefetch hook drained it
        if (t == 0) bulk_store_drain();
        warp_sync();
#pragma unroll
        for (int i = 0; i < MR; ++i)
#pragma unroll
          for (int j = 0; j < NC; ++j) tile[(c.rg + R * i) + (c.cg + G * j) * LD] = a[i][j];
      }
      fence_async_smem();
      warp_sync();
      if (t == 0 && valid) {
        bulk_store(gptr(mat), tile, kBytes);
      }
      if (valid) {
        T *tg = reinterpret_cast<T *>(p.tau) + mat * p.strideT;
        for (int idx = t; idx < c.kmax; idx += GT) tg[idx] = c.taus[idx];
      }
      warp_sync();
      if (qn + gridDim.x < nitems) pending = qn + gridDim.x;
    }
    if (t == 0) bulk_store_drain();
  }

  template <bool ORG>
  static __device__ __forceinline__ void run(const RfArgs &p) {
    if constexpr (GT > 32 && !STAGE && !ORG) {
      run_cta_loop(p);
      return;
    }
    if constexpr (GT <= 32 && GT * GPB == 32 && STAGE && EX && !ORG && Cfg::E == 1) {
      if (p.bulk) {  // contiguous, aligned batch: persistent prefetching loop
        run_warp_loop(p);
        return;
      }
    }
    extern __shared__ __align__(16) float smem[];
    const int tid = threadIdx.x;
    const int grp = tid / GT;
    const int t = tid - grp * GT;
    Ctx c;
    c.t = t;
    c.grp = grp;
    c.rg = t % R;
    c.cg = t / R;
    c.lane = tid & 31;
    c.wid = __shfl_sync(0xffffffffu, t >> 5, 0);
    c.kmax = p.kmax;
    long long mat = (long long)blockIdx.x * GPB + grp;
    const bool active = mat < p.batch;
    if (!active) mat = p.batch - 1;
    float *gs = smem + grp * Cfg::kSmallWords;
    c.vbuf = reinterpret_cast<T *>(gs);
    c.taus = c.vbuf + NBUF * VB;
    T *Ab = reinterpret_cast<T *>(p.A) + mat * p.strideA;
    T a[MR][NC];
    load_matrix(p, c, smem, Ab, mat, active, a);

    if constexpr (ORG) {
      // columns >= k start as the identity (xORG2R initialisation)
#pragma unroll
      for (int i = 0; i < MR; ++i)
#pragma unroll
        for (int j = 0; j < NC; ++j) {
          const int r = c.rg + R * i, col = c.cg + G * j;
          if (col >= p.kmax) a[i][j] = X::sel(r == col, X::one(), X::zero());
        }
      const T *tg = reinterpret_cast<const T *>(p.tau) + mat * p.strideT;
      org_panels<NC - 1>(c, a, p.kmax, tg);
    } else {
      if constexpr (kFullUnroll && EX && GT <= 32) {
        ufactor(c, a);
      } else {
        panels<0>(c, a);
      }
      group_sync<GT, GPB>(grp);  // every tau published before the tau store
    }

    store_matrix(p, c, smem, Ab, mat, active, a);
    // tau list -> global (each tau was published before a group barrier)
    if (!ORG && active) {
      T *tg = reinterpret_cast<T *>(p.tau) + mat * p.strideT;
      for (int idx = t; idx < p.kmax; idx += GT) tg[idx] = c.taus[idx];
    }
  }
};

// MB = minimum resident CTAs per SM (launch bounds): caps the registers per
// thread so that MB groups of a small-matrix class share an SM.  MB = 1
// emits no minimum at all: an explicit ".minnctapersm 1" lets ptxas take
// more registers (e.g. c64 96x96: 198 -> 148 us without it, C3/C4 equal;
// profiles/r01/experiments/ab_launch_bounds.jsonl)
template <class T, int R, int G, int MR, int NC, int GPB, bool STAGE, bool EX, bool AUG, int MB = 1>
__global__ void __launch_bounds__(R * G * GPB, MB > 1 ? MB : 0) geqrf_rf_kernel(const RfArgs p) {
  RfKernel<T, R, G, MR, NC, GPB, STAGE, EX, AUG>::template run<false>(p);
}

// p.kmax = k (reflectors), p.n = columns of Q, p.tau read-only
template <class T, int R, int G, int MR, int NC, int GPB, bool STAGE, bool EX, bool AUG, int MB = 1>
__global__ void __launch_bounds__(R * G * GPB, MB > 1 ? MB : 0) orgqr_rf_kernel(const RfArgs p) {
  RfKernel<T, R, G, MR, NC, GPB, STAGE, EX, AUG>::template run<true>(p);
}

}  // namespace bqr

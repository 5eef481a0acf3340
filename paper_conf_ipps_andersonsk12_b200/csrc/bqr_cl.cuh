// bqr_cl.cuh -- cluster-per-matrix complex Householder QR (the
// §8(a) a9 option; H1/H3: a few large matrices spread over more SMs).
//
// One thread-block CLUSTER of CL CTAs factors one complex64 matrix of up to
// 256 rows and CL*W*NC columns (with up to nrhs right-hand sides appended as
// columns of [A | B]: the fused Q^H B of P:L313).  Every warp of the cluster
// is a column group: lane l holds rows l + 32 i (i < 8) of the columns
// gcg + G s (s < NC, G = CL*W, gcg = rank * W + warp), the 2D-cyclic layout
// of Fig. 6 with 32 row lanes.  Column k's reflector (xLARFG,
// "a square root, two divides, and two multiplies"; LAPACK signs,
// P:L305) is formed by the warp owning column k and published to EVERY CTA
// of the cluster: v (rows < k zero, row k one) and tau are written into each
// CTA's shared vector ring by asynchronous distributed-shared-memory stores
// (st.async ... mbarrier::complete_tx) that count their bytes against that
// CTA's "full" mbarrier, whose one local arrival per phase (thread 0, with
// expect_tx) is made ahead of time.  A release-arrive per CTA instead costs
// a GPU-scope MEMBAR each (90 vs 59 us for one 240 x 66 matrix).
// Consumers wait on their own CTA's barrier, read v from shared memory and
// apply H_k^H = I - conj(tau) v v^H to their columns (w = v^H a, 32-lane
// butterfly; a -= v conj(tau) w).  The owner of column k+1 updates that
// column first and publishes reflector k+1 before its other columns
// (one-column look-ahead).  There is no consumer -> producer signal: the
// owner of column c publishes v_c only after loading v_{c-1}, and every warp
// owns one of any G consecutive columns, so when v_{k+NBUF} (NBUF >= G+1)
// is published every warp has loaded v_k into registers.
#pragma once
#include <cooperative_groups.h>
#include "bqr_common.cuh"

// LAZY: the owner of column k+2 applies v_k to that column only and defers
// the rest of step k until after its look-ahead at step k+1.  Parity green
// but slower on B200 (cl1 86 vs 72 us, cl4 72 vs 60 us at batch 32): the
// owner of k+2 already finishes its remainder while the owner of k+1 runs
// the look-ahead chain, so deferring only moves work (profiles/r02/
// experiments/c4_cluster.jsonl)
#ifndef BQR_CL_LAZY
#define BQR_CL_LAZY 0
#endif
// FUSED: look_fused (one butterfly for the look-ahead dot and the next
// column's norm).  Parity green but slower on B200 (cl4 71.7 vs 61.4 us,
// cl1 73.7 vs 71.7 us at batch 32): off
#ifndef BQR_CL_FFMA2
#define BQR_CL_FFMA2 1
#endif
#ifndef BQR_CL_LOCAL
#define BQR_CL_LOCAL 1
#endif
#ifndef BQR_CL_FUSED
#define BQR_CL_FUSED 0
#endif

namespace bqr {
namespace cl {

struct Args {
  float2 *A;
  float2 *tau;
  float2 *B;  // nullptr when nrhs == 0
  long long batch;
  int m, n, kmax, lda, ldb, nrhs;
  long long strideA, strideT, strideB;
};

template <int CL, int W, int NC>
struct Cfg {
  static constexpr int MR = 8;  // 32 lanes x 8 rows = 256 rows
  static constexpr int MMAX = 32 * MR;
  static constexpr int G = CL * W;
  static constexpr int NMAX = G * NC;
  static constexpr int NBUF = G + 2;
  static constexpr int kThreads = 32 * W;
  static constexpr size_t kVecBytes = (size_t)NBUF * MMAX * 8;
  static constexpr size_t kTauBytes = (size_t)NBUF * 8;
  static constexpr size_t kSmemBytes = kVecBytes + kTauBytes + (size_t)NBUF * 8;
  static constexpr unsigned kStepBytes = MMAX * 8 + 8;  // v and tau, per CTA and step
};

#ifdef BQR_CL_TIMING
// per-step stamps of the look-ahead owner in the first cluster, first matrix
// (clock64 of its SM; with CL = 1 every warp is on one SM): [k][0] v_k
// arrived, [1] dot + update of column k+1 done, [2] norm reduced, [3]
// reflector k+1 published (stores issued)
constexpr int kClDbgSteps = 80;
static __device__ long long g_cl_dbg[kClDbgSteps * 4];
#define CL_STAMP(c, k, e)                                                                  \
  do {                                                                                      \
    if (blockIdx.x < gridDim.x && (c).mat == 0 && (c).lane == 0 && (k) < kClDbgSteps)     \
      g_cl_dbg[(k) * 4 + (e)] = clock64();                                                  \
  } while (0)
#else
#define CL_STAMP(c, k, e) \
  do {                    \
  } while (0)
#endif

__device__ __forceinline__ unsigned cl_smem_u32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }

__device__ __forceinline__ unsigned cl_mapa(unsigned a, unsigned rank) {
  unsigned ra;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(a), "r"(rank));
  return ra;
}
// 8-byte store into a (possibly remote) CTA's shared memory that counts its
// bytes against that CTA's mbarrier (no fence on the producer's chain)
__device__ __forceinline__ void cl_st_async(unsigned raddr, float2 v, unsigned rbar) {
  asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v2.f32 [%0], {%1, %2}, [%3];" ::"r"(raddr),
               "f"(v.x), "f"(v.y), "r"(rbar)
               : "memory");
}
__device__ __forceinline__ void cl_expect(unsigned long long *bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(cl_smem_u32(bar)), "r"(bytes)
               : "memory");
}

__device__ __forceinline__ bool cl_try_wait(unsigned long long *bar, unsigned parity) {
  unsigned ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(cl_smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}

__device__ __forceinline__ float2 cl_allreduce(float2 x) {
#pragma unroll
  for (int o = 16; o >= 1; o >>= 1) {
    x.x += __shfl_xor_sync(0xffffffffu, x.x, o);
    x.y += __shfl_xor_sync(0xffffffffu, x.y, o);
  }
  return x;
}

template <int CL, int W, int NC>
struct Kernel {
  using C = Cfg<CL, W, NC>;
  using X = El<float2>;
  static constexpr int MR = C::MR, G = C::G, NBUF = C::NBUF;
  // a one-CTA "cluster" publishes with shared stores + a release.cta arrive
  // per lane (count 32) instead of st.async + expect_tx
  static constexpr bool kLocal = CL == 1 && BQR_CL_LOCAL;
  using Tile = float2[MR][NC];

  struct Ctx {
    float2 *vbuf;  // [NBUF][MMAX] local
    float2 *tbuf;  // [NBUF] local
    unsigned long long *full;
    int lane, gcg;
    int gbase;
    long long mat;
    const Args *p;
  };

  // reflector of column k (slot S of this warp) and its publication to every
  // CTA of the cluster (ring entry gbase + k); tau also to global memory
  template <int S>
  static __device__ __forceinline__ void reflect_publish(Ctx &c, Tile &a, int k) {
    const int kl = k & 31, ki = k >> 5;
    float2 xa = a[0][S];
#pragma unroll
    for (int i = 1; i < MR; ++i)
      if (i == ki) xa = a[i][S];
    const float2 alpha = X::shfl(xa, kl);
    float sg = 0.f;
#pragma unroll
    for (int i = 0; i < MR; ++i) {
      const int r = c.lane + 32 * i;
      sg = r > k ? X::abs2_acc(a[i][S], sg) : sg;
    }
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) sg += __shfl_xor_sync(0xffffffffu, sg, o);
    CL_STAMP(c, k - 1 < 0 ? 0 : k - 1, 2);
    publish<S>(c, a, k, alpha, sg);
    CL_STAMP(c, k - 1 < 0 ? 0 : k - 1, 3);
  }

  // xLARFG from alpha and sigma = sum_{r>k} |a_rk|^2, column k (slot S)
  // scaled in place, v and tau published
  template <int S>
  static __device__ __forceinline__ void publish(Ctx &c, Tile &a, int k, float2 alpha, float sg) {
    const Reflector<float2> h = make_reflector(alpha, sg);
    float2 v[MR];
#pragma unroll
    for (int i = 0; i < MR; ++i) {
      const int r = c.lane + 32 * i;
      const float2 xs = X::mul(a[i][S], h.scal);
      v[i] = r > k ? xs : (r == k ? X::one() : X::zero());
      a[i][S] = r > k ? xs : (r == k ? make_float2(h.beta, 0.f) : a[i][S]);
    }
    const int b = (c.gbase + k) % NBUF;
    if constexpr (kLocal) {
      // one CTA: plain shared stores, each lane's arrive (release.cta) covers them
#pragma unroll
      for (int i = 0; i < MR; ++i) c.vbuf[b * C::MMAX + c.lane + 32 * i] = v[i];
      if (c.lane == 0) c.tbuf[b] = h.tau;
      __syncwarp();
      asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(cl_smem_u32(c.full + b)) : "memory");
    } else {
      const unsigned va = cl_smem_u32(c.vbuf + b * C::MMAX + c.lane), ta = cl_smem_u32(c.tbuf + b),
                     ba = cl_smem_u32(c.full + b);
#pragma unroll
      for (int q = 0; q < CL; ++q) {
        const unsigned rv = cl_mapa(va, (unsigned)q), rb = cl_mapa(ba, (unsigned)q);
#pragma unroll
        for (int i = 0; i < MR; ++i) cl_st_async(rv + 256u * i, v[i], rb);
        if (c.lane == 0) cl_st_async(cl_mapa(ta, (unsigned)q), h.tau, rb);
      }
    }
    if (c.lane == 0) c.p->tau[c.mat * c.p->strideT + k] = h.tau;
  }

  // look-ahead on column k1 (slot S) fused with its norm: one butterfly of
  // w = v^H a together with the pre-update sums over rows r > k1 of |a|^2,
  // conj(v) a and |v|^2, from which sigma' = sum |a - v t|^2 (t = conj(tau) w)
  // = saa - 2 Re(conj(t) sva) + |t|^2 svv.  Heavy cancellation
  // (sigma' < saa / 4) falls back to the direct sum after the update.
  template <int S>
  static __device__ __forceinline__ void look_fused(Ctx &c, Tile &a, const float2 (&v)[MR], float2 ct, int k1) {
    const int kl = k1 & 31, ki = k1 >> 5;
    float r6[6] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f};  // w.x w.y saa sva.x sva.y svv
    float2 xa = a[0][S], xv = v[0];
#pragma unroll
    for (int i = 0; i < MR; ++i) {
      const int r = c.lane + 32 * i;
      const float2 x = a[i][S], y = v[i];
      const float2 w = X::cfma(y, x, make_float2(r6[0], r6[1]));
      r6[0] = w.x;
      r6[1] = w.y;
      if (i > 0 && i == ki) {
        xa = x;
        xv = y;
      }
      if (r > k1) {
        r6[2] = X::abs2_acc(x, r6[2]);
        const float2 q = X::cfma(y, x, make_float2(r6[3], r6[4]));
        r6[3] = q.x;
        r6[4] = q.y;
        r6[5] = X::abs2_acc(y, r6[5]);
      }
    }
    const float2 alpha0 = X::shfl(xa, kl), v0 = X::shfl(xv, kl);
    row_allreduce_multi<32, 6>(r6, c.lane);
    const float2 tw = X::mul(ct, make_float2(r6[0], r6[1]));
#pragma unroll
    for (int i = 0; i < MR; ++i) a[i][S] = X::fnms(v[i], tw, a[i][S]);
    const float2 alpha = X::fnms(v0, tw, alpha0);
    // Re(conj(t) sva) = t.x sva.x + t.y sva.y
    const float cross = fmaf(tw.x, r6[3], tw.y * r6[4]);
    const float t2 = fmaf(tw.x, tw.x, tw.y * tw.y);
    float sg = fmaf(t2, r6[5], fmaf(-2.f, cross, r6[2]));
    if (!(sg >= 0.25f * r6[2])) {
      sg = 0.f;
#pragma unroll
      for (int i = 0; i < MR; ++i) {
        const int r = c.lane + 32 * i;
        sg = r > k1 ? X::abs2_acc(a[i][S], sg) : sg;
      }
#pragma unroll
      for (int o = 16; o >= 1; o >>= 1) sg += __shfl_xor_sync(0xffffffffu, sg, o);
    }
    publish<S>(c, a, k1, alpha, sg);
  }

  // packed complex arithmetic (FFMA2 on the (re, im) pair with a broadcast
  // scalar): conj(v) a summed as P = sum vr (ar, ai), Q = sum vi (ar, ai),
  // w = (P.x + Q.y, P.y - Q.x); a - v t = a + vr (-tr, -ti) + vi (ti, -tr)
  template <int S>
  static __device__ __forceinline__ float2 dotS(const float2 (&v)[MR], const Tile &a) {
#if BQR_CL_FFMA2
    float2 P = X::zero(), Q = X::zero();
#pragma unroll
    for (int i = 0; i < MR; ++i) {
      P = __ffma2_rn(make_float2(v[i].x, v[i].x), a[i][S], P);
      Q = __ffma2_rn(make_float2(v[i].y, v[i].y), a[i][S], Q);
    }
    return make_float2(P.x + Q.y, P.y - Q.x);
#else
    float2 w = X::zero();
#pragma unroll
    for (int i = 0; i < MR; ++i) w = X::cfma(v[i], a[i][S], w);
    return w;
#endif
  }
  template <int S>
  static __device__ __forceinline__ void updS(const float2 (&v)[MR], float2 tw, Tile &a) {
#if BQR_CL_FFMA2
    const float2 n1 = make_float2(-tw.x, -tw.y), n2 = make_float2(tw.y, -tw.x);
#pragma unroll
    for (int i = 0; i < MR; ++i) {
      a[i][S] = __ffma2_rn(make_float2(v[i].x, v[i].x), n1, a[i][S]);
      a[i][S] = __ffma2_rn(make_float2(v[i].y, v[i].y), n2, a[i][S]);
    }
#else
#pragma unroll
    for (int i = 0; i < MR; ++i) a[i][S] = X::fnms(v[i], tw, a[i][S]);
#endif
  }

  static __device__ __forceinline__ float2 dot_slot(const float2 (&v)[MR], const Tile &a, int s) {
#if BQR_CL_FFMA2
    float2 P = X::zero(), Q = X::zero();
#pragma unroll
    for (int i = 0; i < MR; ++i) {
      P = __ffma2_rn(make_float2(v[i].x, v[i].x), a[i][s], P);
      Q = __ffma2_rn(make_float2(v[i].y, v[i].y), a[i][s], Q);
    }
    return make_float2(P.x + Q.y, P.y - Q.x);
#else
    float2 w = X::zero();
#pragma unroll
    for (int i = 0; i < MR; ++i) w = X::cfma(v[i], a[i][s], w);
    return w;
#endif
  }
  static __device__ __forceinline__ void upd_slot(const float2 (&v)[MR], float2 tw, Tile &a, int s) {
#if BQR_CL_FFMA2
    const float2 n1 = make_float2(-tw.x, -tw.y), n2 = make_float2(tw.y, -tw.x);
#pragma unroll
    for (int i = 0; i < MR; ++i) {
      a[i][s] = __ffma2_rn(make_float2(v[i].x, v[i].x), n1, a[i][s]);
      a[i][s] = __ffma2_rn(make_float2(v[i].y, v[i].y), n2, a[i][s]);
    }
#else
#pragma unroll
    for (int i = 0; i < MR; ++i) a[i][s] = X::fnms(v[i], tw, a[i][s]);
#endif
  }

  // a -= v conj(tau) (v^H a) on slot S
  template <int S>
  static __device__ __forceinline__ void apply1(Tile &a, const float2 (&v)[MR], float2 ct) {
    float2 w = dotS<S>(v, a);
    w = cl_allreduce(w);
    const float2 tw = X::mul(ct, w);
    updS<S>(v, tw, a);
#ifdef BQR_CL_TIMING
    if (threadIdx.x % 32 == 0) asm volatile("" ::"f"(a[0][S].x), "f"(a[MR - 1][S].y));
#endif
  }

  // H_kk^H on every live slot of this warp (column > kk, < ncol, != excl),
  // slots below S0 hold no such column
  template <int S0>
  static __device__ __forceinline__ void rest(Ctx &c, Tile &a, const float2 (&v)[MR], float2 ct, int kk, int excl,
                                              int ncol) {
    // only slots S0 .. NC-1 can hold live columns: reduce just those
    constexpr int NL = NC - S0;
    float wv[2 * NL];
#pragma unroll
    for (int j = 0; j < NL; ++j) {
      const float2 w = dot_slot(v, a, S0 + j);
      wv[2 * j] = w.x;
      wv[2 * j + 1] = w.y;
    }
    row_allreduce_multi<32, 2 * NL>(wv, c.lane);
#pragma unroll
    for (int j = 0; j < NL; ++j) {
      const int s = S0 + j;
      const int col = c.gcg + G * s;
      if (col > kk && col < ncol && col != excl) {
        const float2 tw = X::mul(ct, make_float2(wv[2 * j], wv[2 * j + 1]));
        upd_slot(v, tw, a, s);
      }
    }
  }

  // H_k^H on column kc only (its slot is S0 or S0 + 1)
  template <int S0>
  static __device__ __forceinline__ void apply_col(Tile &a, const float2 (&v)[MR], float2 ct, int kc) {
    if (kc / G != S0) {
      if constexpr (S0 + 1 < NC) apply1<S0 + 1>(a, v, ct);
    } else {
      apply1<S0>(a, v, ct);
    }
  }

  // step k (pivot slot S0 of its owner): wait for v_k; the owner of column
  // k+1 updates it and publishes reflector k+1 (look-ahead), then every
  // warp applies v_k to its other columns (with BQR_CL_LAZY, the owner of
  // column k+2 defers that remainder past its own look-ahead at step k+1).
  template <int S0>
  static __device__ __forceinline__ void step(Ctx &c, Tile &a, int k, int ncol, float2 (&vd)[MR], float2 &ctd,
                                              bool &defer) {
    const int g = c.gbase + k;
    const int b = g % NBUF;
    while (!cl_try_wait(c.full + b, (unsigned)(g / NBUF) & 1u)) {
    }
    float2 v[MR];
#pragma unroll
    for (int i = 0; i < MR; ++i) v[i] = c.vbuf[b * C::MMAX + c.lane + 32 * i];
    const float2 ct = X::conj(c.tbuf[b]);
    // the local arrival of ring entry g + NBUF - 1 (its previous phase, g - 1,
    // has completed: this warp waited for it)
    if (!kLocal && threadIdx.x == 0 && k + NBUF - 1 < c.p->kmax) cl_expect(c.full + (g + NBUF - 1) % NBUF, C::kStepBytes);
    const int k1 = k + 1, k2 = k + 2;
    const bool look = k1 < c.p->kmax && c.gcg == k1 % G;
    if (look) {
      CL_STAMP(c, k, 0);
      if (k1 / G != S0) {
        if constexpr (S0 + 1 < NC) {
#if BQR_CL_FUSED
          look_fused<S0 + 1>(c, a, v, ct, k1);
#else
          apply1<S0 + 1>(a, v, ct);
          CL_STAMP(c, k, 1);
          reflect_publish<S0 + 1>(c, a, k1);
#endif
        }
      } else {
#if BQR_CL_FUSED
        look_fused<S0>(c, a, v, ct, k1);
#else
        apply1<S0>(a, v, ct);
        CL_STAMP(c, k, 1);
        reflect_publish<S0>(c, a, k1);
#endif
      }
    }
#if BQR_CL_LAZY
    if (!look && k2 < c.p->kmax && c.gcg == k2 % G) {
      apply_col<S0>(a, v, ct, k2);
#pragma unroll
      for (int i = 0; i < MR; ++i) vd[i] = v[i];
      ctd = ct;
      defer = true;
      return;
    }
    if (defer) {
      rest<S0>(c, a, vd, ctd, k - 1, k1, ncol);
      defer = false;
    }
#endif
    rest<S0>(c, a, v, ct, k, look ? k1 : -1, ncol);
  }

  template <int S0>
  static __device__ __forceinline__ void sweep(Ctx &c, Tile &a, int ncol, float2 (&vd)[MR], float2 &ctd, bool &defer) {
    if constexpr (S0 < NC) {
#pragma unroll 1
      for (int r0 = 0; r0 < G; ++r0) {
        const int k = S0 * G + r0;
        if (k >= c.p->kmax) return;
        step<S0>(c, a, k, ncol, vd, ctd, defer);
      }
      sweep<S0 + 1>(c, a, ncol, vd, ctd, defer);
    }
  }

  static __device__ __forceinline__ void run(const Args &p) {
    extern __shared__ __align__(16) unsigned char smem_cl[];
    namespace cg = cooperative_groups;
    cg::cluster_group cluster = cg::this_cluster();
    Ctx c;
    c.vbuf = reinterpret_cast<float2 *>(smem_cl);
    c.tbuf = reinterpret_cast<float2 *>(smem_cl + C::kVecBytes);
    c.full = reinterpret_cast<unsigned long long *>(smem_cl + C::kVecBytes + C::kTauBytes);
    c.lane = threadIdx.x & 31;
    const int wid = __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0);
    const unsigned rank = cluster.block_rank();
    c.gcg = (int)rank * W + wid;
    c.p = &p;
    c.gbase = 0;
    if (threadIdx.x < NBUF) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(cl_smem_u32(c.full + threadIdx.x)), "r"(kLocal ? 32 : 1)
                   : "memory");
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    cluster.sync();
    const long long nclus = gridDim.x / CL;
    const int ncol = p.n + p.nrhs;
    for (long long mat = blockIdx.x / CL; mat < p.batch; mat += nclus) {
      c.mat = mat;
      const float2 *Am = p.A + mat * p.strideA;
      const float2 *Bm = p.nrhs > 0 ? p.B + mat * p.strideB : nullptr;
      Tile a;
#pragma unroll
      for (int s = 0; s < NC; ++s) {
        const int col = c.gcg + G * s;
#pragma unroll
        for (int i = 0; i < MR; ++i) {
          const int r = c.lane + 32 * i;
          float2 x = X::zero();
          if (r < p.m) {
            if (col < p.n) x = Am[r + (long long)col * p.lda];
            else if (col < ncol) x = Bm[r + (long long)(col - p.n) * p.ldb];
          }
          a[i][s] = x;
        }
      }
      if (!kLocal && threadIdx.x == 0)
        for (int j = 0; j < NBUF - 1 && j < p.kmax; ++j) cl_expect(c.full + (c.gbase + j) % NBUF, C::kStepBytes);
      if (c.gcg == 0 && p.kmax > 0) reflect_publish<0>(c, a, 0);
      float2 vd[MR];
      float2 ctd = X::zero();
      bool defer = false;
#pragma unroll
      for (int i = 0; i < MR; ++i) vd[i] = X::zero();
      sweep<0>(c, a, ncol, vd, ctd, defer);
#pragma unroll
      for (int s = 0; s < NC; ++s) {
        const int col = c.gcg + G * s;
        float2 *dst = col < p.n ? p.A + mat * p.strideA + (long long)col * p.lda
                                : (col < ncol ? p.B + mat * p.strideB + (long long)(col - p.n) * p.ldb : nullptr);
        if (dst) {
#pragma unroll
          for (int i = 0; i < MR; ++i) {
            const int r = c.lane + 32 * i;
            if (r < p.m) dst[r] = a[i][s];
          }
        }
      }
      c.gbase += p.kmax;
      // no CTA reuses a ring entry (or exits) while a peer may still write it
      cluster.sync();
    }
  }
};

template <int CL, int W, int NC>
__global__ void __cluster_dims__(CL, 1, 1) __launch_bounds__(32 * W, 1) geqrf_cl_kernel(const Args p) {
  Kernel<CL, W, NC>::run(p);
}

}  // namespace cl
}  // namespace bqr

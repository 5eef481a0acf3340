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
//     matrix-vector product -- is a warp shuffle butterfly, no barrier, no
//     thread-0 serial loop) and columns are cyclic over the G column groups;
//     R and G need not be equal (the paper needed p = sqrt(p)^2);
//   * a group is a sub-warp (several matrices per warp, e.g. 2 x 56x56 fp32
//     per warp), a warp, or a CTA (e.g. 240x66 c64 across 16 warps);
//   * the reflector is computed redundantly by every lane of the owning
//     column group with IEEE sqrt/div (north star; not the 22-bit hardware
//     path of P:L321); its vector is published through a double-buffered
//     shared-memory slot, so ONE group barrier per column suffices;
//   * the compile-time panel recursion advances the first live
//     register row/column slot per panel, so finished rows/columns cost
//     nothing; inside a panel the column loop is a runtime loop (small code);
//   * global <-> register staging either directly (row lanes >= 8: each warp
//     access is a contiguous column segment) or through a bank-conflict-free
//     padded shared-memory tile filled by 16-byte cp.async (small R).
#pragma once
#include "bqr_common.cuh"

namespace bqr {

struct RfArgs {
  void *A;
  void *tau;
  long long batch;
  int lda, m, n, kmax;
  int ldS;        // staging tile leading dimension (elements)
  int tileWords;  // staging tile stride per group (32-bit words)
  int vec4;       // 16-byte vectorised staging legal (lda%4==0, m%4==0, aligned)
};

template <int GT, int GPB>
__device__ __forceinline__ void group_sync(int grp) {
  if constexpr (GT <= 32) {
    __syncwarp();
  } else if constexpr (GPB == 1) {
    __syncthreads();
  } else {
    asm volatile("bar.sync %0, %1;" ::"r"(1 + grp), "r"(GT) : "memory");
  }
}

__device__ __forceinline__ void cp_async16(void *smem_dst, const void *gmem_src) {
  unsigned s = (unsigned)__cvta_generic_to_shared(smem_dst);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem_src) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() {
  asm volatile("cp.async.wait_all;\n" ::: "memory");
}

template <class T, int R, int G, int MR, int NC, int GPB, bool STAGE>
struct RfCfg {
  static constexpr int GT = R * G;
  static constexpr int NT = GT * GPB;
  static constexpr int MMAX = R * MR;
  static constexpr int NMAX = G * NC;
  static constexpr int E = sizeof(T) / 4;
  // per-group small smem: double-buffered Householder vector + tau list
  static constexpr int kSmallWords = (2 * MMAX + NMAX) * E;
  static constexpr int kSmallAll = ((GPB * kSmallWords + 31) / 32) * 32;
  static_assert(R >= 1 && R <= 32 && (R & (R - 1)) == 0, "R must be a power of two <= 32");
  static_assert(GT <= 32 ? (32 % GT == 0) : (GT % 32 == 0), "group must tile warps");
  static_assert(!STAGE || E == 1, "smem staging implemented for fp32");
  // rows that may equal the pivot row inside one panel (see column())
  static constexpr int NMASK = (G + R - 1) / R + 1;
};

template <class T, int R, int G, int MR, int NC, int GPB, bool STAGE>
struct RfKernel {
  using Cfg = RfCfg<T, R, G, MR, NC, GPB, STAGE>;
  using X = El<T>;
  static constexpr int GT = Cfg::GT;
  static constexpr int MMAX = Cfg::MMAX;

  struct Ctx {
    T *vbuf;   // [2][MMAX]
    T *taus;   // [NMAX]
    int rg, cg, t, lane, grp;
    int kmax;
  };

  // One Householder step on column k (panel P, first live register row I0).
  template <int P, int I0>
  static __device__ __forceinline__ void column(Ctx &c, T (&a)[MR][NC], int k) {
    const int kk = k - P * G;  // owning column group
    T *vb = c.vbuf + (k & 1) * MMAX;
    // ---- reflector (xLARFG) on the owning column group: Table VI "Column"
    bool warp_has_owner;
    if constexpr (GT <= 32) {
      warp_has_owner = true;
    } else {
      warp_has_owner = (kk / (32 / R)) == (c.t >> 5);
    }
    if (warp_has_owner) {
      float sig = 0.f;
      T alpha = X::zero();
#pragma unroll
      for (int i = I0; i < MR; ++i) {
        const int r = c.rg + R * i;
        const T x = a[i][P];
        if (i < I0 + Cfg::NMASK) {
          sig = X::abs2_acc(X::sel(r > k, x, X::zero()), sig);
          alpha = X::sel(r == k, x, alpha);
        } else {
          sig = X::abs2_acc(x, sig);
        }
      }
      sig = row_allreduce_f<R>(sig);
      if constexpr (R > 1) alpha = X::shfl(alpha, (c.lane & ~(R - 1)) | (k & (R - 1)));
      const Reflector<T> h = make_reflector(alpha, sig);
      if (c.cg == kk) {
        // scale x, write beta, publish v (v_k = 1, v_r = 0 above the pivot)
#pragma unroll
        for (int i = I0; i < MR; ++i) {
          const int r = c.rg + R * i;
          T x = a[i][P];
          T v;
          if (i < I0 + Cfg::NMASK) {
            const T xs = X::mul(x, h.scal);
            v = X::sel(r > k, xs, X::sel(r == k, X::one(), X::zero()));
            x = X::sel(r > k, xs, X::sel(r == k, X::make(h.beta, 0.f), x));
          } else {
            v = X::mul(x, h.scal);
            x = v;
          }
          a[i][P] = x;
          vb[r] = v;
        }
        if (c.rg == 0) c.taus[k] = h.tau;
      }
    }
    group_sync<GT, GPB>(c.grp);
    // ---- trailing update: Table VI "Trailing Matrix" (Listing 7)
    const T ct = X::conj(c.taus[k]);
    T v[MR];
#pragma unroll
    for (int i = I0; i < MR; ++i) v[i] = vb[c.rg + R * i];
    T tw[NC];
#pragma unroll
    for (int j = P; j < NC; ++j) {
      T w = X::zero();
#pragma unroll
      for (int i = I0; i < MR; ++i) w = X::cfma(v[i], a[i][j], w);
      w = row_allreduce<R>(w);
      tw[j] = X::mul(ct, w);
      if (j == P) tw[j] = X::sel(c.cg > kk, tw[j], X::zero());
    }
#pragma unroll
    for (int j = P; j < NC; ++j) {
#pragma unroll
      for (int i = I0; i < MR; ++i) a[i][j] = X::fnms(v[i], tw[j], a[i][j]);
    }
  }

  template <int P>
  static __device__ __forceinline__ void panels(Ctx &c, T (&a)[MR][NC]) {
    if constexpr (P < NC) {
      constexpr int I0 = (P * G) / R;
      const int kbeg = P * G;
      if (kbeg >= c.kmax) return;
      const int kend = min(kbeg + G, c.kmax);
#pragma unroll 1
      for (int k = kbeg; k < kend; ++k) column<P, I0>(c, a, k);
      panels<P + 1>(c, a);
    }
  }

  // ---- xORG2R / xUNG2R: Q = H_0 ... H_{k-1} applied backwards (i = k-1 .. 0)
  template <int P, int I0>
  static __device__ __forceinline__ void org_column(Ctx &c, T (&a)[MR][NC], int i, const T *tau_g) {
    const int kk = i - P * G;
    T *vb = c.vbuf + (i & 1) * MMAX;
    const T ti = tau_g[i];
    if (c.cg == kk) {
#pragma unroll
      for (int ii = I0; ii < MR; ++ii) {
        const int r = c.rg + R * ii;
        vb[r] = X::sel(r > i, a[ii][P], X::sel(r == i, X::one(), X::zero()));
      }
    }
    group_sync<GT, GPB>(c.grp);
    T v[MR];
#pragma unroll
    for (int ii = I0; ii < MR; ++ii) v[ii] = vb[c.rg + R * ii];
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

  template <bool ORG>
  static __device__ __forceinline__ void run(const RfArgs &p) {
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
    c.kmax = p.kmax;
    long long mat = (long long)blockIdx.x * GPB + grp;
    const bool active = mat < p.batch;
    if (!active) mat = p.batch - 1;
    float *gs = smem + grp * Cfg::kSmallWords;
    c.vbuf = reinterpret_cast<T *>(gs);
    c.taus = c.vbuf + 2 * MMAX;
    T *Ab = reinterpret_cast<T *>(p.A) + mat * (long long)p.lda * p.n;
    const int m = p.m, n = p.n;
    T a[MR][NC];
    if constexpr (STAGE) {
      float *tile = smem + Cfg::kSmallAll + grp * p.tileWords;
      const float *Ag = reinterpret_cast<const float *>(Ab);
      if (active) {
        if (p.vec4) {
          const int mq = m >> 2;
          const int nch = mq * n;
          for (int q = t; q < nch; q += GT) {
            const int col = q / mq, rr = (q - col * mq) << 2;
            cp_async16(tile + rr + col * p.ldS, Ag + rr + (long long)col * p.lda);
          }
          cp_async_wait_all();
        } else {
          const int nch = m * n;
          for (int q = t; q < nch; q += GT) {
            const int col = q / m, rr = q - col * m;
            tile[rr + col * p.ldS] = Ag[rr + (long long)col * p.lda];
          }
        }
      }
      group_sync<GT, GPB>(grp);
#pragma unroll
      for (int i = 0; i < MR; ++i)
#pragma unroll
        for (int j = 0; j < NC; ++j) {
          const int r = c.rg + R * i, col = c.cg + G * j;
          a[i][j] = (active && r < m && col < n) ? tile[r + col * p.ldS] : 0.f;
        }
    } else {
#pragma unroll
      for (int i = 0; i < MR; ++i)
#pragma unroll
        for (int j = 0; j < NC; ++j) {
          const int r = c.rg + R * i, col = c.cg + G * j;
          a[i][j] = (active && r < m && col < n) ? Ab[r + (long long)col * p.lda] : X::zero();
        }
    }

    if constexpr (ORG) {
      // columns >= k start as the identity (xORG2R initialisation)
#pragma unroll
      for (int i = 0; i < MR; ++i)
#pragma unroll
        for (int j = 0; j < NC; ++j) {
          const int r = c.rg + R * i, col = c.cg + G * j;
          if (col >= p.kmax) a[i][j] = X::sel(r == col, X::one(), X::zero());
        }
      const T *tg = reinterpret_cast<const T *>(p.tau) + mat * (long long)p.kmax;
      org_panels<NC - 1>(c, a, p.kmax, tg);
    } else {
      panels<0>(c, a);
    }

    if constexpr (STAGE) {
      float *tile = smem + Cfg::kSmallAll + grp * p.tileWords;
      float *Ag = reinterpret_cast<float *>(Ab);
#pragma unroll
      for (int i = 0; i < MR; ++i)
#pragma unroll
        for (int j = 0; j < NC; ++j) {
          const int r = c.rg + R * i, col = c.cg + G * j;
          if (r < m && col < n) tile[r + col * p.ldS] = a[i][j];
        }
      group_sync<GT, GPB>(grp);
      if (active) {
        if (p.vec4) {
          const int mq = m >> 2;
          const int nch = mq * n;
          for (int q = t; q < nch; q += GT) {
            const int col = q / mq, rr = (q - col * mq) << 2;
            *reinterpret_cast<float4 *>(Ag + rr + (long long)col * p.lda) =
                *reinterpret_cast<const float4 *>(tile + rr + col * p.ldS);
          }
        } else {
          const int nch = m * n;
          for (int q = t; q < nch; q += GT) {
            const int col = q / m, rr = q - col * m;
            Ag[rr + (long long)col * p.lda] = tile[rr + col * p.ldS];
          }
        }
      }
    } else if (active) {
#pragma unroll
      for (int i = 0; i < MR; ++i)
#pragma unroll
        for (int j = 0; j < NC; ++j) {
          const int r = c.rg + R * i, col = c.cg + G * j;
          if (r < m && col < n) Ab[r + (long long)col * p.lda] = a[i][j];
        }
    }
    // tau list -> global (taus complete: every column ended with a group sync)
    if (!ORG && active) {
      T *tg = reinterpret_cast<T *>(p.tau) + mat * (long long)p.kmax;
      for (int idx = t; idx < p.kmax; idx += GT) tg[idx] = c.taus[idx];
    }
  }
};

template <class T, int R, int G, int MR, int NC, int GPB, bool STAGE>
__global__ void __launch_bounds__(R * G * GPB) geqrf_rf_kernel(const RfArgs p) {
  RfKernel<T, R, G, MR, NC, GPB, STAGE>::template run<false>(p);
}

// p.kmax = k (reflectors), p.n = columns of Q, p.tau read-only
template <class T, int R, int G, int MR, int NC, int GPB, bool STAGE>
__global__ void __launch_bounds__(R * G * GPB) orgqr_rf_kernel(const RfArgs p) {
  RfKernel<T, R, G, MR, NC, GPB, STAGE>::template run<true>(p);
}

}  // namespace bqr

// bqr_co.cuh -- "column-owner" register-file Householder QR for small real
// matrices (the C3 headline class, 56x56 fp32), one matrix per 14-28 lanes.
//
// Same method as bqr_rf.cuh (Sec. V; per column "norm ->
// square root, two divides, two multiplies -> scale -> matrix-vector product
// -> rank-1 update", Table VI), different mapping:
//   * a lane owns WHOLE columns (L column lanes, column j on lane j mod L,
//     slot j div L), split over only H in {1, 2, 4} row lanes (rows
//     interleaved by quads: lane h holds rows 4(H r + h) .. +3 of quad r).
//     With H = 1 the matrix-vector product and the column norm need no
//     cross-lane reduction at all; with H = 2 / 4 one or two shuffle levels.
//     (The paper's square sqrt(p) x sqrt(p) grid, Fig. 6, and the R x G grid
//     of bqr_rf.cuh reduce over R = 4..32 row lanes every column.)
//   * the matrix-vector product and the rank-1 update run on row pairs with
//     packed FP32 (fma.rn.f32x2 = SASS FFMA2), v is a 16-byte shared-memory
//     broadcast (LDS.128), the reflector scalar is an FFMA2 broadcast operand;
//   * look-ahead: in step k the column lanes first apply H_k to the slot that
//     holds column k+1, every lane forms the reflector of its copy of that
//     slot (branch-free; only the owner's bits are kept), then H_k is applied
//     to the remaining slots while the sqrt/div chain is in flight, and only
//     then does the owner publish v_{k+1} (so no shared-memory store sits
//     between the loads of the rest-update and the reflector arithmetic);
//   * compile-time panels of PW columns (PW | L) fix the live slot range and
//     the first live row quad; inside a panel the column loop is a runtime
//     loop, which keeps the code inside the instruction cache;
//   * one warp = MPW = 32 / (H LS) matrices, independent persistent warps:
//     TMA bulk prefetch (cp.async.bulk + mbarrier) of the warp's next
//     matrices into shared memory while the current ones are factored,
//     16-byte register <-> global stores of the result.
// Dead lanes of a partially live slot apply the reflector with a zero scalar
// (a + v * 0): the value is unchanged except that an exact -0.0 entry of a
// finished column may come back as +0.0 (numerically equal).
#pragma once
#include "bqr_common.cuh"
#include "bqr_rf.cuh"

namespace bqr {

struct CoArgs {
  float *A;
  float *tau;
  long long batch;
};

__device__ __forceinline__ void sts128_if(float *p, float4 v, bool on) {
  asm volatile(
      "{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %5, 0;\n\t"
      "@q st.shared.v4.f32 [%0], {%1, %2, %3, %4};\n}" ::"r"(smem_u32(p)),
      "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w), "r"((int)on)
      : "memory");
}
__device__ __forceinline__ void sts32_if(float *p, float v, bool on) {
  asm volatile(
      "{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %2, 0;\n\t"
      "@q st.shared.f32 [%0], %1;\n}" ::"r"(smem_u32(p)),
      "f"(v), "r"((int)on)
      : "memory");
}

template <int M, int N, int L, int H, int LS, int PW>
struct CoCfg {
  static constexpr int MPW = 32 / (H * LS);   // matrices per warp
  static constexpr int S = (N + L - 1) / L;   // column slots per lane
  static constexpr int NQ = M / (4 * H);      // row quads per lane
  static constexpr int VBW = M + 4;           // vector buffer: rows [0, M), tau at [M]
  static constexpr int TILE_F = MPW * M * N;  // prefetch tile (floats)
  static constexpr int MAT_F = 2 * VBW + ((3 * N + 3) / 4) * 4;  // vector buffers + meta (beta, scale, tau)
  static constexpr int WARP_F = TILE_F + MPW * MAT_F + 4;
  static constexpr int WPC = 4;               // independent warps per CTA (one per SMSP)
  static constexpr int NPANEL = (N + PW - 1) / PW;
  static constexpr size_t SMEM = (size_t)WPC * WARP_F * 4;
  static_assert(H == 1 || H == 2 || H == 4, "H row lanes");
  static_assert(L <= LS && H * LS <= 32 && 32 % (H * LS) == 0, "lane mapping");
  static_assert(L % PW == 0, "a panel stays inside one column slot");
  static_assert(M % (4 * H) == 0 && M >= N, "row quads, tall or square");
  static_assert(WARP_F % 4 == 0 && VBW % 4 == 0 && MAT_F % 4 == 0, "16-byte alignment");
};

template <int M, int N, int L, int H, int LS, int PW>
struct CoKernel {
  using C = CoCfg<M, N, L, H, LS, PW>;
  static constexpr int S = C::S, NQ = C::NQ, VBW = C::VBW, MPW = C::MPW;

  struct Ctx {
    float *vb;     // this matrix's two vector buffers
    int c;         // column lane (clamped to L-1 on idle lanes)
    int h;         // row lane
    int lane;
    bool lane_ok;  // not an idle lane
  };

  static __device__ __forceinline__ int row_of(const Ctx &x, int r, int e) { return (H * r + x.h) * 4 + e; }
  static __device__ __forceinline__ float el(const float2 (&qd)[2], int e) {
    return e == 0 ? qd[0].x : e == 1 ? qd[0].y : e == 2 ? qd[1].x : qd[1].y;
  }
  static __device__ __forceinline__ void set_el(float2 (&qd)[2], int e, float v) {
    if (e == 0) qd[0].x = v;
    else if (e == 1) qd[0].y = v;
    else if (e == 2) qd[1].x = v;
    else qd[1].y = v;
  }
  // sum over the H row lanes of a column
  static __device__ __forceinline__ float hsum(float v) {
    if constexpr (H >= 2) v += __shfl_xor_sync(0xffffffffu, v, LS);
    if constexpr (H >= 4) v += __shfl_xor_sync(0xffffffffu, v, 2 * LS);
    return v;
  }
  static __device__ __forceinline__ float2 lo(const float4 &v) { return make_float2(v.x, v.y); }
  static __device__ __forceinline__ float2 hi(const float4 &v) { return make_float2(v.z, v.w); }

  // One column step: apply H_{j-1} (APPLY) and form reflector j.  The
  // owner's column keeps its unscaled entries in the registers (x, alpha on
  // the diagonal); beta and the scale 1/(alpha - beta) go to the matrix's
  // meta arrays and are applied once, when the column is stored.
  template <int P, bool APPLY>
  static __device__ __forceinline__ void step(const Ctx &x, float2 (&a)[S][NQ][2], int j) {
    constexpr int JLO = PW * P;
    constexpr int JHI = (PW * P + PW < N) ? PW * P + PW : N;
    constexpr int S1 = JLO / L;                       // slot holding columns [JLO, JHI)
    constexpr int R0 = JLO > 0 ? JLO - 1 : 0;         // lowest live row in this panel
    constexpr int Q0 = R0 / (4 * H);                  // first live quad (conservative)
    constexpr int QM = (JHI + 4 * H - 1) / (4 * H);   // quads below QM may hold rows <= j
    const int k = j - 1;
    float tau_k = 0.f;
    const float *vk = x.vb + (k & 1) * VBW;
    if constexpr (APPLY) {
      tau_k = lds32(vk + M);
      // (a5/a6 on the look-ahead slot) w = v^T a, a -= tau w v
      float2 p0 = make_float2(0.f, 0.f);
#pragma unroll
      for (int r = Q0; r < NQ; ++r) {
        const float4 v = lds128(vk + (H * r + x.h) * 4);
        p0 = __ffma2_rn(lo(v), a[S1][r][0], p0);
        p0 = __ffma2_rn(hi(v), a[S1][r][1], p0);
      }
      const float w = hsum(p0.x + p0.y);
      const int col = L * S1 + x.c;
      const float nt = (col > k && col < N) ? -(tau_k * w) : 0.f;
      const float2 nt2 = make_float2(nt, nt);
#pragma unroll
      for (int r = Q0; r < NQ; ++r) {
        const float4 v = lds128(vk + (H * r + x.h) * 4);
        a[S1][r][0] = __ffma2_rn(lo(v), nt2, a[S1][r][0]);
        a[S1][r][1] = __ffma2_rn(hi(v), nt2, a[S1][r][1]);
      }
    }
    // (a2/a3) reflector of column j from this lane's copy of slot S1
    // row (H r + h) 4 + e  vs  j  <=>  compile-time 4 H r + e  vs  dj = j - 4 h
    const int dj = j - 4 * x.h;
    float sig = 0.f, alpha_m = 0.f;
    float2 sg0 = make_float2(0.f, 0.f);
#pragma unroll
    for (int r = Q0; r < NQ; ++r) {
      if (r < QM) {
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const float xe = el(a[S1][r], e);
          alpha_m = (4 * H * r + e == dj) ? xe : alpha_m;
          const float xm = (4 * H * r + e > dj) ? xe : 0.f;
          sig = fmaf(xm, xm, sig);
        }
      } else {
        sg0 = __ffma2_rn(a[S1][r][0], a[S1][r][0], sg0);
        sg0 = __ffma2_rn(a[S1][r][1], a[S1][r][1], sg0);
      }
    }
    sig = hsum(sig + (sg0.x + sg0.y));
    float alpha = alpha_m;
    if constexpr (H > 1) {
      const int hj = (j >> 2) % H;
      const int src = (x.lane & ~(H * LS - 1)) | (hj * LS) | (x.lane & (LS - 1));
      alpha = __shfl_sync(0xffffffffu, alpha_m, src);
    }
    const Reflector<float> hr = make_reflector(alpha, sig);
    const bool owner = x.lane_ok && (x.c == j - L * S1);
    // (a5/a6) H_k on the remaining slots, independent of the reflector chain
    if constexpr (APPLY && S1 + 1 < S) {
      constexpr int NS = S - S1 - 1;
      float2 acc[NS];
#pragma unroll
      for (int s = 0; s < NS; ++s) acc[s] = make_float2(0.f, 0.f);
#pragma unroll
      for (int r = Q0; r < NQ; ++r) {
        const float4 v = lds128(vk + (H * r + x.h) * 4);
#pragma unroll
        for (int s = 0; s < NS; ++s) {
          acc[s] = __ffma2_rn(lo(v), a[S1 + 1 + s][r][0], acc[s]);
          acc[s] = __ffma2_rn(hi(v), a[S1 + 1 + s][r][1], acc[s]);
        }
      }
      float nt[NS];
#pragma unroll
      for (int s = 0; s < NS; ++s) {
        const float w = hsum(acc[s].x + acc[s].y);
        const int col = L * (S1 + 1 + s) + x.c;
        nt[s] = col < N ? -(tau_k * w) : 0.f;
      }
#pragma unroll
      for (int r = Q0; r < NQ; ++r) {
        const float4 v = lds128(vk + (H * r + x.h) * 4);
#pragma unroll
        for (int s = 0; s < NS; ++s) {
          const float2 n2 = make_float2(nt[s], nt[s]);
          a[S1 + 1 + s][r][0] = __ffma2_rn(lo(v), n2, a[S1 + 1 + s][r][0]);
          a[S1 + 1 + s][r][1] = __ffma2_rn(hi(v), n2, a[S1 + 1 + s][r][1]);
        }
      }
    }
    // (a4) publish v_j = x / (alpha - beta) below the pivot, 1 on it, 0 above.
    // Buffer j&1 held v_{j-2}: rows < j-2 are already 0, so the owner writes
    // the scaled quads that start at row >= j-3 and then rows j-3..j
    // (0, 0, 0, 1) over them.  Predicated stores, no branch (a divergent
    // region here makes the compiler guard every later shuffle).
    float *vj = x.vb + (j & 1) * VBW;
    const float2 sc2 = make_float2(hr.scal, hr.scal);
#pragma unroll
    for (int r = Q0; r < NQ; ++r) {
      const float2 u0 = __fmul2_rn(a[S1][r][0], sc2), u1 = __fmul2_rn(a[S1][r][1], sc2);
      const bool on = r >= QM || 4 * H * r >= dj - 3;
      sts128_if(vj + (H * r + x.h) * 4, make_float4(u0.x, u0.y, u1.x, u1.y), owner && on);
    }
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const int i = j - 3 + e;
      const bool mine = i >= 0 && ((i >> 2) % H) == x.h;
      sts32_if(vj + (i >= 0 ? i : 0), e == 3 ? 1.f : 0.f, owner && mine);
    }
    float *meta = x.vb + 2 * VBW;
    sts32_if(vj + M, hr.tau, owner && x.h == 0);
    sts32_if(meta + j, hr.beta, owner && x.h == 0);
    sts32_if(meta + N + j, hr.scal, owner && x.h == 0);
    sts32_if(meta + 2 * N + j, hr.tau, owner && x.h == 0);
    warp_sync();
  }

  template <int P>
  static __device__ __forceinline__ void panels(const Ctx &x, float2 (&a)[S][NQ][2]) {
    constexpr int JLO = PW * P;
    constexpr int JHI = (PW * P + PW < N) ? PW * P + PW : N;
    int j0 = JLO;
    if constexpr (P == 0) {
      step<0, false>(x, a, 0);
      j0 = 1;
    }
#pragma unroll 1
    for (int j = j0; j < JHI; ++j) step<P, true>(x, a, j);
    if constexpr (P + 1 < C::NPANEL) panels<P + 1>(x, a);
  }

  static __device__ __forceinline__ void run(const CoArgs &p) {
    extern __shared__ __align__(16) float smem[];
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    float *ws = smem + w * C::WARP_F;
    float *tile = ws;
    void *bar = ws + C::TILE_F + MPW * C::MAT_F;
    const int q = lane / (H * LS);
    const int craw = lane % LS;
    Ctx x;
    x.h = (lane / LS) % H;
    x.c = craw < L ? craw : L - 1;
    x.lane = lane;
    x.lane_ok = craw < L;
    x.vb = ws + C::TILE_F + q * C::MAT_F;
    const float *meta = x.vb + 2 * VBW;
    const long long items = (p.batch + MPW - 1) / MPW;
    long long item = (long long)blockIdx.x * C::WPC + w;
    const long long stride = (long long)gridDim.x * C::WPC;
    if (lane == 0) mbar_init(bar, 1);
    warp_sync();
    if (item >= items) return;
    auto issue = [&](long long it) {
      const long long m0 = it * MPW;
      const long long nm = p.batch - m0 < MPW ? p.batch - m0 : MPW;
      bulk_load(tile, p.A + m0 * (M * N), (unsigned)(nm * (M * N * 4)), bar);
    };
    if (lane == 0) issue(item);
    unsigned phase = 0;
#pragma unroll 1
    for (; item < items; item += stride) {
      while (!mbar_try_wait(bar, phase)) {
      }
      phase ^= 1;
      float2 a[S][NQ][2];
      const float *tq = tile + q * (M * N);
#pragma unroll
      for (int s = 0; s < S; ++s) {
        const int col = L * s + x.c;
#pragma unroll
        for (int r = 0; r < NQ; ++r) {
          float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
          if (col < N) v = *reinterpret_cast<const float4 *>(tq + col * M + (H * r + x.h) * 4);
          a[s][r][0] = lo(v);
          a[s][r][1] = hi(v);
        }
      }
      warp_sync();
      const long long nxt = item + stride;
      if (lane == 0 && nxt < items) {
        fence_async_smem();
        issue(nxt);
      }
      panels<0>(x, a);
      // (a7) store [R; V]: column j = R above the pivot, beta on it, x * scale below
      const long long mat = item * MPW + q;
      if (mat < p.batch && x.lane_ok) {
        float *Ag = p.A + mat * (M * N);
#pragma unroll
        for (int s = 0; s < S; ++s) {
          const int col = L * s + x.c;
          if (col < N) {
            const float beta = meta[col], sc = meta[N + col];
            const int dc = col - 4 * x.h;
#pragma unroll
            for (int r = 0; r < NQ; ++r) {
              float o[4];
#pragma unroll
              for (int e = 0; e < 4; ++e) {
                const float xe = el(a[s][r], e);
                const int b = 4 * H * r + e;
                o[e] = b > dc ? xe * sc : (b == dc ? beta : xe);
              }
              *reinterpret_cast<float4 *>(Ag + col * M + (H * r + x.h) * 4) = make_float4(o[0], o[1], o[2], o[3]);
            }
            if (x.h == 0) p.tau[mat * N + col] = meta[2 * N + col];
          }
        }
      }
      warp_sync();  // meta arrays reused by the next matrix
    }
  }
};

template <int M, int N, int L, int H, int LS, int PW, int MINB>
__global__ void __launch_bounds__(128, MINB) geqrf_co_kernel(const CoArgs p) {
  CoKernel<M, N, L, H, LS, PW>::run(p);
}

}  // namespace bqr

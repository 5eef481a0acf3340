// bqr_tiny_apply.cu -- thread-per-matrix plans (n <= 8), the Q^H B kernel
// dispatch and the IEEE-math self-test kernel.
#include "bqr_launch.cuh"

namespace bqr {
namespace host {

namespace {
// tiny exact sizes 1 <= n <= m <= 8
template <class T, int M>
Plan tiny_plan_n(int n) {
  switch (n) {
#define TN(NN) \
  case NN:     \
    if constexpr (NN <= M) return Plan{"tiny", &launch_tiny<T, M, NN>, nullptr}; break;
    TN(1) TN(2) TN(3) TN(4) TN(5) TN(6) TN(7) TN(8)
#undef TN
  }
  return Plan{nullptr, nullptr, nullptr};
}

template <class T>
Plan tiny_plan(int m, int n) {
  switch (m) {
    case 1: return tiny_plan_n<T, 1>(n);
    case 2: return tiny_plan_n<T, 2>(n);
    case 3: return tiny_plan_n<T, 3>(n);
    case 4: return tiny_plan_n<T, 4>(n);
    case 5: return tiny_plan_n<T, 5>(n);
    case 6: return tiny_plan_n<T, 6>(n);
    case 7: return tiny_plan_n<T, 7>(n);
    case 8: return tiny_plan_n<T, 8>(n);
  }
  return Plan{nullptr, nullptr, nullptr};
}

// self-test of the branch-free IEEE helpers (bqr_common.cuh) against the
// CUDA library's sqrt.rn / div.rn on random normal operands spanning the
// exponent range the contract (reading Q6) can produce, plus subnormal
// operands (the FTZ guard).
__device__ __forceinline__ unsigned hash32(unsigned x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
  return x;
}
__device__ __forceinline__ float rand_normal_float(unsigned h, int emin, int emax) {
  const unsigned mant = h & 0x7fffffU;
  const int e = emin + (int)((h >> 23) % (unsigned)(emax - emin + 1));
  return __uint_as_float(((unsigned)(e + 127) << 23) | mant);
}
__global__ void selftest_math_kernel(long long n, unsigned seed, unsigned long long *counts) {
  unsigned long long bad_sqrt = 0, bad_div = 0, bad_rcp = 0, bad_sub = 0;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    const unsigned h1 = hash32((unsigned)i * 2654435761U ^ seed), h2 = hash32(h1 ^ 0x9e3779b9U);
    const float x = rand_normal_float(h1, -100, 100);           // sigma / |z|^2 range
    const float a = rand_normal_float(h2, -50, 50) * ((h2 & 1) ? -1.f : 1.f);
    const float b = rand_normal_float(h1 ^ h2, -50, 50) * ((h1 & 2) ? -1.f : 1.f);
    bad_sqrt += __float_as_uint(bqr::sqrt_rn(x)) != __float_as_uint(__fsqrt_rn(x));
    bad_div += __float_as_uint(bqr::div_rn(a, b)) != __float_as_uint(__fdiv_rn(a, b));
    bad_rcp += __float_as_uint(bqr::div_rn(1.0f, b)) != __float_as_uint(__frcp_rn(b));
    // subnormal operands of the square root (the FTZ guard)
    const float xs = __uint_as_float((h1 & 0x7fffffU) | 1u);  // nonzero (sqrt_rn(0) is the caller's skip case)
    bad_sub += __float_as_uint(bqr::sqrt_rn(xs)) != __float_as_uint(__fsqrt_rn(xs));
  }
  atomicAdd(&counts[0], bad_sqrt);
  atomicAdd(&counts[1], bad_div);
  atomicAdd(&counts[2], bad_rcp);
  atomicAdd(&counts[3], bad_sub);
}

template <class T>
int launch_apply_views(const void *A, int lda, long long sA, const void *tau, long long sT, void *B, int ldb,
                       long long sB, int m, int k, int nrhs, long long batch, cudaStream_t s) {
  ApplyArgs a{A, tau, B, batch, lda, 0, m, k, nrhs, ldb, sA, sT, sB};
  return apply_dispatch<T>(a, s);
}

}  // namespace

Plan tiny_plan_f32(int m, int n) { return tiny_plan<float>(m, n); }
Plan tiny_plan_c64(int m, int n) { return tiny_plan<float2>(m, n); }
int apply_dispatch_f32(const ApplyArgs &a, cudaStream_t s) { return apply_dispatch<float>(a, s); }
int apply_dispatch_c64(const ApplyArgs &a, cudaStream_t s) { return apply_dispatch<float2>(a, s); }
int launch_selftest_math(long long n, unsigned seed, unsigned long long *counts, cudaStream_t s) {
  selftest_math_kernel<<<1184, 256, 0, s>>>(n, seed, counts);
  return finish_launch();
}

}  // namespace host
}  // namespace bqr

// Microbenchmarks (NEXT-4 / SURVEY B12): FP32 FMA issue throughput on sm_100a
// for the operand patterns of the Householder kernels, FFMA vs packed FFMA2,
// and the latencies that bound the per-column chain.
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ float2 ffma2(float2 a, float2 b, float2 c) {
  unsigned long long A = *reinterpret_cast<unsigned long long*>(&a), B = *reinterpret_cast<unsigned long long*>(&b),
                     C = *reinterpret_cast<unsigned long long*>(&c), D;
  asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(D) : "l"(A), "l"(B), "l"(C));
  return *reinterpret_cast<float2*>(&D);
}

// rank-1 update pattern: a[i] = fma(-v[i], t, a[i]) over 32 registers
template <int N>
__global__ void k_rank1(float *out, int iters, float t) {
  float a[N], v[N];
#pragma unroll
  for (int i = 0; i < N; ++i) { a[i] = threadIdx.x * 0.001f + i; v[i] = 0.5f + i * 1e-3f; }
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < N; ++i) a[i] = fmaf(-v[i], t, a[i]);
    t = t * 0.999f;
  }
  float s = 0;
#pragma unroll
  for (int i = 0; i < N; ++i) s += a[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template <int N>
__global__ void k_rank1_x2(float *out, int iters, float t) {
  float2 a[N / 2], v[N / 2];
#pragma unroll
  for (int i = 0; i < N / 2; ++i) { a[i] = make_float2(threadIdx.x * 0.001f + i, i); v[i] = make_float2(0.5f + i * 1e-3f, 0.25f); }
  for (int it = 0; it < iters; ++it) {
    float2 nt = make_float2(-t, -t);
#pragma unroll
    for (int i = 0; i < N / 2; ++i) a[i] = ffma2(v[i], nt, a[i]);
    t = t * 0.999f;
  }
  float s = 0;
#pragma unroll
  for (int i = 0; i < N / 2; ++i) s += a[i].x + a[i].y;
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
// dependent chain latency
__global__ void k_chain(float *out, long long *cyc, int iters) {
  float x = threadIdx.x * 1e-3f;
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 16; ++j) x = fmaf(x, 0.9999f, 1e-6f);
  }
  long long t1 = clock64();
  out[threadIdx.x] = x;
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
}
__global__ void k_shfl_chain(float *out, long long *cyc, int iters) {
  float x = threadIdx.x * 1e-3f;
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 16; ++j) x = __shfl_xor_sync(0xffffffffu, x, 1) + 1e-6f;
  }
  long long t1 = clock64();
  out[threadIdx.x] = x;
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
}
__global__ void k_lds_chain(float *out, long long *cyc, int iters) {
  __shared__ int buf[1024];
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) buf[i] = (i + 1) & 1023;
  __syncthreads();
  int p = threadIdx.x;
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 16; ++j) p = buf[p];
  }
  long long t1 = clock64();
  out[threadIdx.x] = p;
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
}
__global__ void k_sqrtdiv_chain(float *out, long long *cyc, int iters) {
  float x = 2.0f + threadIdx.x;
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 8; ++j) x = __fdiv_rn(1.0f, __fsqrt_rn(x)) + 1.5f;
  }
  long long t1 = clock64();
  out[threadIdx.x] = x;
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
}

int main() {
  int dev = 0, sms = 0, clk = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
  float *out; long long *cyc;
  cudaMalloc(&out, 1 << 26); cudaMalloc(&cyc, 64);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const int iters = 20000;
  // warm
  k_rank1<32><<<sms * 8, 256>>>(out, 100, 1.0f);
  cudaDeviceSynchronize();
  for (int wps = 4; wps <= 32; wps *= 2) {  // warps per SM
    float ms;
    cudaEventRecord(e0);
    k_rank1<32><<<sms * (wps / 8 > 0 ? wps / 8 : 1), wps >= 8 ? 256 : wps * 32>>>(out, iters, 1.0f);
    cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
    double fma = (double)sms * wps * 32 * 32.0 * iters;
    printf("{\"bench\":\"ffma_rank1\",\"warps_per_sm\":%d,\"tflops\":%.2f,\"fma_per_clk_sm_at_max\":%.1f}\n", wps,
           2 * fma / ms / 1e9, fma / (ms * 1e-3) / sms / (1965e6));
    cudaEventRecord(e0);
    k_rank1_x2<32><<<sms * (wps / 8 > 0 ? wps / 8 : 1), wps >= 8 ? 256 : wps * 32>>>(out, iters, 1.0f);
    cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
    printf("{\"bench\":\"ffma2_rank1\",\"warps_per_sm\":%d,\"tflops\":%.2f,\"fma_per_clk_sm_at_max\":%.1f}\n", wps,
           2 * fma / ms / 1e9, fma / (ms * 1e-3) / sms / (1965e6));
  }
  long long h;
  k_chain<<<1, 32>>>(out, cyc, 1000); cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
  printf("{\"bench\":\"ffma_dep_latency_cycles\",\"value\":%.2f}\n", h / (1000.0 * 16));
  k_shfl_chain<<<1, 32>>>(out, cyc, 1000); cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
  printf("{\"bench\":\"shfl_plus_fadd_dep_latency_cycles\",\"value\":%.2f}\n", h / (1000.0 * 16));
  k_lds_chain<<<1, 32>>>(out, cyc, 1000); cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
  printf("{\"bench\":\"lds_dep_latency_cycles\",\"value\":%.2f}\n", h / (1000.0 * 16));
  k_sqrtdiv_chain<<<1, 32>>>(out, cyc, 1000); cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
  printf("{\"bench\":\"sqrt_rn_div_rn_fadd_chain_cycles\",\"value\":%.2f}\n", h / (1000.0 * 8));
  printf("{\"sms\":%d,\"clock_khz\":%d}\n", sms, clk);
  return 0;
}

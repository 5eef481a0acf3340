// PCIe zero-copy bandwidth of SM loads/stores on pinned (UVA-mapped) host
// memory: a grid-stride copy host -> device, device -> host and both at once
// (16-byte coalesced accesses), against cudaMemcpyAsync on the copy engines.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void copy4(const float4 *__restrict__ src, float4 *__restrict__ dst, long long n) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
    dst[i] = src[i];
}
__global__ void copy_both(const float4 *__restrict__ hin, float4 *__restrict__ din, const float4 *__restrict__ dout,
                          float4 *__restrict__ hout, long long n) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    din[i] = hin[i];
    hout[i] = dout[i];
  }
}
int main() {
  const size_t bytes = 62720000;
  const long long n = bytes / 16;
  float4 *h1, *h2, *d1, *d2;
  cudaHostAlloc(&h1, bytes, cudaHostAllocDefault);
  cudaHostAlloc(&h2, bytes, cudaHostAllocDefault);
  cudaMalloc(&d1, bytes);
  cudaMalloc(&d2, bytes);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  auto time = [&](auto f) {
    for (int i = 0; i < 3; ++i) f();
    cudaEventRecord(a);
    for (int i = 0; i < 10; ++i) f();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    return ms / 10;
  };
  for (int g : {148, 296, 592, 1184}) {
    float t1 = time([&] { copy4<<<g, 512>>>(h1, d1, n); });
    float t2 = time([&] { copy4<<<g, 512>>>(d2, h2, n); });
    float t3 = time([&] { copy_both<<<g, 512>>>(h1, d1, d2, h2, n); });
    printf("{\"grid\": %d, \"h2d_gbs\": %.1f, \"d2h_gbs\": %.1f, \"both_gbs_total\": %.1f}\n", g, bytes / t1 / 1e6,
           bytes / t2 / 1e6, 2 * bytes / t3 / 1e6);
  }
  float tc = time([&] { cudaMemcpyAsync(d1, h1, bytes, cudaMemcpyHostToDevice); });
  printf("{\"memcpy_h2d_gbs\": %.1f}\n", bytes / tc / 1e6);
  return 0;
}

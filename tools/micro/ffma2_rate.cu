// Issue rate of packed FFMA2 vs scalar FFMA for 1..4 warps per SM
// sub-partition (clock64 cycles per warp instruction, 8 independent chains).
#include <cstdio>
#include <cuda_runtime.h>
template <bool PK>
__global__ void k(float *out, long long *cyc, int iters) {
  float2 a[8];
  float s[8];
  for (int i = 0; i < 8; ++i) { a[i] = make_float2(threadIdx.x * 1e-3f + i, i * 0.5f); s[i] = a[i].x; }
  // register operands (3-register forms): values the compiler cannot fold
  const float2 m = make_float2(1.0001f + out[0] * 1e-30f, 0.9999f + out[1] * 1e-30f);
  const float2 d = make_float2(1e-6f + out[2] * 1e-30f, -1e-6f + out[3] * 1e-30f);
  const float ms = m.x, ds = d.x;
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (PK) a[i] = __ffma2_rn(a[i], m, d);
      else s[i] = fmaf(s[i], ms, ds);
    }
  }
  long long t1 = clock64();
  float acc = 0.f;
  for (int i = 0; i < 8; ++i) acc += PK ? a[i].x + a[i].y : s[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
int main() {
  float *out; long long *cyc; cudaMalloc(&out, 1 << 20); cudaMemset(out, 0, 1 << 20); cudaMalloc(&cyc, 1 << 16);
  const int iters = 4096;
  for (int pk = 0; pk < 2; ++pk)
    for (int w : {1, 2, 4, 8, 16}) {
      long long h = 0;
      if (pk) k<true><<<1, 32 * w>>>(out, cyc, iters); else k<false><<<1, 32 * w>>>(out, cyc, iters);
      if (pk) k<true><<<1, 32 * w>>>(out, cyc, iters); else k<false><<<1, 32 * w>>>(out, cyc, iters);
      cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
      const double instr = (double)iters * 8 * w;  // warp instructions in the SM
      printf("{\"op\": \"%s\", \"warps_per_sm\": %d, \"cycles\": %lld, \"cyc_per_warp_instr_per_sm\": %.3f, \"fma_per_clk_per_sm\": %.1f}\n",
             pk ? "FFMA2" : "FFMA", w, h, h / instr, instr * 32 * (pk ? 2 : 1) / h);
    }
  return 0;
}

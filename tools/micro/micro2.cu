// B200 (sm_100a) microbenchmarks, round 2 (NEXT-4; the paper's
// Sec. II: Tables II-IV, Fig. 2).
//
// All rates are in SM clock cycles measured inside the kernel (clock64), so
// they do not depend on the DVFS clock the box happens to run at.
//   * FP32 pipe: FFMA vs packed FFMA2 for the operand patterns of the
//     Householder kernels (rank-1 update with a reused v / a broadcast scalar,
//     dot-product accumulation), FMA per clock per SM;
//   * shared memory: LDS.128 bandwidth (bytes/clk/SM), the paper's Table II
//     analogue; LDS pointer-chase latency (Table III);
//   * synchronisation: __syncthreads vs threads (Fig. 2 / Table IV alpha_sync),
//     named barrier, mbarrier arrive->wait between two warps, cluster barrier,
//     DSMEM remote load latency;
//   * shuffle + add latency, FFMA latency, IEEE sqrt+div chain.
// Output: one JSON object per line.
#include <cooperative_groups.h>
#include <cstdio>
#include <cuda_runtime.h>

namespace cg = cooperative_groups;

__device__ __forceinline__ float2 ffma2(float2 a, float2 b, float2 c) {
  return __ffma2_rn(a, b, c);
}

__device__ unsigned long long g_cyc[4096];

#define TIMED_BEGIN                \
  __syncthreads();                 \
  long long t0 = clock64();
#define TIMED_END                                                   \
  __syncthreads();                                                  \
  long long t1 = clock64();                                         \
  if (threadIdx.x == 0) g_cyc[blockIdx.x % 4096] = (unsigned long long)(t1 - t0);

// ---------------------------------------------------------------- FP32 pipe
// A: scalar FFMA rank-1, v[p] reused across 4 columns j, t[j] per column
__global__ void k_ffma_rank1(float *out, int iters) {
  float a[4][16], v[16], t[4];
#pragma unroll
  for (int p = 0; p < 16; ++p) v[p] = 0.5f + p * 1e-3f + threadIdx.x * 1e-6f;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    t[j] = 1e-3f * (j + 1) + threadIdx.x * 1e-7f;
#pragma unroll
    for (int p = 0; p < 16; ++p) a[j][p] = threadIdx.x * 1e-3f + p + j;
  }
  TIMED_BEGIN
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int p = 0; p < 16; ++p)
#pragma unroll
      for (int j = 0; j < 4; ++j) a[j][p] = fmaf(-v[p], t[j], a[j][p]);
#pragma unroll
    for (int j = 0; j < 4; ++j) t[j] *= 0.999f;
  }
  TIMED_END
  float s = 0;
#pragma unroll
  for (int j = 0; j < 4; ++j)
#pragma unroll
    for (int p = 0; p < 16; ++p) s += a[j][p];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
// B: FFMA2 rank-1 on row pairs, v pair reused across j, broadcast scalar t[j]
__global__ void k_ffma2_rank1(float *out, int iters) {
  float2 a[4][8], v[8];
  float t[4];
#pragma unroll
  for (int p = 0; p < 8; ++p) v[p] = make_float2(0.5f + p * 1e-3f + threadIdx.x * 1e-6f, 0.25f + p * 1e-3f);
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    t[j] = 1e-3f * (j + 1) + threadIdx.x * 1e-7f;
#pragma unroll
    for (int p = 0; p < 8; ++p) a[j][p] = make_float2(threadIdx.x * 1e-3f + p + j, p - j);
  }
  TIMED_BEGIN
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int p = 0; p < 8; ++p)
#pragma unroll
      for (int j = 0; j < 4; ++j) a[j][p] = ffma2(v[p], make_float2(-t[j], -t[j]), a[j][p]);
#pragma unroll
    for (int j = 0; j < 4; ++j) t[j] *= 0.999f;
  }
  TIMED_END
  float s = 0;
#pragma unroll
  for (int j = 0; j < 4; ++j)
#pragma unroll
    for (int p = 0; p < 8; ++p) s += a[j][p].x + a[j][p].y;
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
// C: FFMA2 rank-1, column-major order (t reused, v pair distinct per row)
__global__ void k_ffma2_rank1_col(float *out, int iters) {
  float2 a[4][8], v[8];
  float t[4];
#pragma unroll
  for (int p = 0; p < 8; ++p) v[p] = make_float2(0.5f + p * 1e-3f + threadIdx.x * 1e-6f, 0.25f + p * 1e-3f);
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    t[j] = 1e-3f * (j + 1) + threadIdx.x * 1e-7f;
#pragma unroll
    for (int p = 0; p < 8; ++p) a[j][p] = make_float2(threadIdx.x * 1e-3f + p + j, p - j);
  }
  TIMED_BEGIN
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 4; ++j)
#pragma unroll
      for (int p = 0; p < 8; ++p) a[j][p] = ffma2(v[p], make_float2(-t[j], -t[j]), a[j][p]);
#pragma unroll
    for (int j = 0; j < 4; ++j) t[j] *= 0.999f;
  }
  TIMED_END
  float s = 0;
#pragma unroll
  for (int j = 0; j < 4; ++j)
#pragma unroll
    for (int p = 0; p < 8; ++p) s += a[j][p].x + a[j][p].y;
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
// D: FFMA2 dot products: acc[j] += v[p] * a[j][p] (v reused over j)
__global__ void k_ffma2_dot(float *out, int iters) {
  float2 a[4][8], v[8], acc[4];
#pragma unroll
  for (int p = 0; p < 8; ++p) v[p] = make_float2(0.5f + p * 1e-3f + threadIdx.x * 1e-6f, 0.25f + p * 1e-3f);
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    acc[j] = make_float2(0.f, 0.f);
#pragma unroll
    for (int p = 0; p < 8; ++p) a[j][p] = make_float2(threadIdx.x * 1e-3f + p + j, p - j);
  }
  TIMED_BEGIN
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int p = 0; p < 8; ++p)
#pragma unroll
      for (int j = 0; j < 4; ++j) acc[j] = ffma2(v[p], a[j][p], acc[j]);
#pragma unroll
    for (int p = 0; p < 8; ++p) v[p].x *= 0.999f;
  }
  TIMED_END
  float s = 0;
#pragma unroll
  for (int j = 0; j < 4; ++j) s += acc[j].x + acc[j].y;
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
// E: scalar FFMA dot products
__global__ void k_ffma_dot(float *out, int iters) {
  float a[4][16], v[16], acc[4][2];
#pragma unroll
  for (int p = 0; p < 16; ++p) v[p] = 0.5f + p * 1e-3f + threadIdx.x * 1e-6f;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    acc[j][0] = acc[j][1] = 0.f;
#pragma unroll
    for (int p = 0; p < 16; ++p) a[j][p] = threadIdx.x * 1e-3f + p + j;
  }
  TIMED_BEGIN
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int p = 0; p < 16; ++p)
#pragma unroll
      for (int j = 0; j < 4; ++j) acc[j][p & 1] = fmaf(v[p], a[j][p], acc[j][p & 1]);
#pragma unroll
    for (int p = 0; p < 16; ++p) v[p] *= 0.999f;
  }
  TIMED_END
  float s = 0;
#pragma unroll
  for (int j = 0; j < 4; ++j) s += acc[j][0] + acc[j][1];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

// ---------------------------------------------------------------- shared memory
__global__ void k_lds_bw(float *out, int iters) {
  __shared__ float4 buf[2048];
  for (int i = threadIdx.x; i < 2048; i += blockDim.x) buf[i] = make_float4(i, i + 1, i + 2, i + 3);
  float4 acc = make_float4(0, 0, 0, 0);
  int base = threadIdx.x;
  TIMED_BEGIN
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      float4 x = buf[(base + 256 * j) & 2047];
      acc.x += x.x;
      acc.y += x.y;
      acc.z += x.z;
      acc.w += x.w;
    }
    base += 32;
  }
  TIMED_END
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc.x + acc.y + acc.z + acc.w;
}

// ---------------------------------------------------------------- latency chains (one warp)
__global__ void k_lat(float *out, long long *cyc, int iters, int which) {
  __shared__ int buf[1024];
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) buf[i] = (i + 33) & 1023;
  __syncthreads();
  float x = 2.0f + threadIdx.x * 1e-3f;
  int p = threadIdx.x;
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 16; ++j) {
      if (which == 0) x = fmaf(x, 0.9999f, 1e-6f);
      else if (which == 1) x = __shfl_xor_sync(0xffffffffu, x, 1) + 1e-6f;
      else if (which == 2) p = buf[p];
      else x = __fdiv_rn(1.0f, __fsqrt_rn(x)) + 1.5f;
    }
  }
  long long t1 = clock64();
  out[threadIdx.x] = x + p;
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
}

// ---------------------------------------------------------------- barriers
__global__ void k_bar(float *out, long long *cyc, int iters) {
  float x = threadIdx.x;
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    __syncthreads();
    x += 1.0f;
  }
  long long t1 = clock64();
  out[blockIdx.x * blockDim.x + threadIdx.x] = x;
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
}
// named barrier among the first `cnt` threads (multiple of 32)
__global__ void k_named_bar(float *out, long long *cyc, int iters, int cnt) {
  float x = threadIdx.x;
  __syncthreads();
  long long t0 = clock64();
  if (threadIdx.x < cnt) {
    for (int it = 0; it < iters; ++it) {
      asm volatile("bar.sync 3, %0;" ::"r"(cnt) : "memory");
      x += 1.0f;
    }
  }
  long long t1 = clock64();
  out[blockIdx.x * blockDim.x + threadIdx.x] = x;
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
}

__device__ __forceinline__ unsigned smem_u32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(void *bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(void *bar) {
  asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(void *bar, unsigned parity) {
  unsigned ok = 0;
  while (!ok) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
  }
}
// ping-pong between warp 0 and warp 1 through two mbarriers (count 1 each):
// one round trip = two arrive->wait hand-offs
__global__ void k_mbar_pingpong(float *out, long long *cyc, int iters) {
  __shared__ __align__(8) unsigned long long bar[2];
  if (threadIdx.x == 0) {
    mbar_init(&bar[0], 1);
    mbar_init(&bar[1], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    const unsigned ph = it & 1;
    if (w == 0) {
      if (lane == 0) mbar_arrive(&bar[0]);
      mbar_wait(&bar[1], ph);
    } else {
      mbar_wait(&bar[0], ph);
      if (lane == 0) mbar_arrive(&bar[1]);
    }
  }
  long long t1 = clock64();
  out[threadIdx.x] = (float)t1;
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
}

// cluster barrier and DSMEM remote-load latency (cluster dims set at launch)
__global__ void k_cluster_bar(float *out, long long *cyc, int iters) {
  cg::cluster_group cl = cg::this_cluster();
  float x = threadIdx.x;
  cl.sync();
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    asm volatile("barrier.cluster.arrive.release;\n\tbarrier.cluster.wait.acquire;" ::: "memory");
    x += 1.0f;
  }
  long long t1 = clock64();
  out[blockIdx.x * blockDim.x + threadIdx.x] = x;
  if (threadIdx.x == 0 && cl.block_rank() == 0) cyc[0] = t1 - t0;
}
__global__ void k_dsmem_chase(float *out, long long *cyc, int iters) {
  __shared__ int buf[1024];
  cg::cluster_group cl = cg::this_cluster();
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) buf[i] = (i + 33) & 1023;
  cl.sync();
  const unsigned peer = (cl.block_rank() + 1) % cl.num_blocks();
  int *rb = cl.map_shared_rank(buf, peer);
  int p = threadIdx.x;
  long long t0 = clock64();
  if (cl.block_rank() == 0 && threadIdx.x == 0) {
    for (int it = 0; it < iters; ++it) {
#pragma unroll
      for (int j = 0; j < 16; ++j) p = rb[p];
    }
  }
  long long t1 = clock64();
  cl.sync();
  out[blockIdx.x * blockDim.x + threadIdx.x] = p;
  if (threadIdx.x == 0 && cl.block_rank() == 0) cyc[0] = t1 - t0;
}

// ---------------------------------------------------------------- launch overhead
__global__ void k_empty(float *out) {
  if (out && threadIdx.x == 1023) out[0] = 0.f;
}

// ---------------------------------------------------------------- host
static unsigned long long max_cyc(int nblk) {
  static unsigned long long h[4096];
  cudaMemcpyFromSymbol(h, g_cyc, sizeof(unsigned long long) * (nblk < 4096 ? nblk : 4096));
  unsigned long long m = 0;
  for (int i = 0; i < nblk && i < 4096; ++i) m = h[i] > m ? h[i] : m;
  return m;
}

typedef void (*KFn)(float *, int);

static void fma_bench(const char *name, KFn k, int sms, float *out, double fma_per_thread_iter) {
  const int iters = 4000;
  for (int wps = 4; wps <= 32; wps *= 2) {
    const int threads = 128, bps = wps / 4;
    k<<<sms * bps, threads>>>(out, 10);
    cudaDeviceSynchronize();
    k<<<sms * bps, threads>>>(out, iters);
    cudaDeviceSynchronize();
    const unsigned long long c = max_cyc(sms * bps);
    const double fma_sm = (double)wps * 32 * fma_per_thread_iter * iters;
    printf("{\"bench\":\"%s\",\"warps_per_sm\":%d,\"fma_per_clk_sm\":%.1f}\n", name, wps, fma_sm / (double)c);
  }
}

int main() {
  int sms = 0, clk = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  float *out;
  long long *cyc;
  cudaMalloc(&out, 1 << 26);
  cudaMalloc(&cyc, 64);
  fma_bench("ffma_rank1_vreuse", k_ffma_rank1, sms, out, 64);
  fma_bench("ffma2_rank1_vreuse_bcast", k_ffma2_rank1, sms, out, 64);
  fma_bench("ffma2_rank1_colmajor_bcast", k_ffma2_rank1_col, sms, out, 64);
  fma_bench("ffma2_dot", k_ffma2_dot, sms, out, 64);
  fma_bench("ffma_dot", k_ffma_dot, sms, out, 64);
  {  // shared-memory bandwidth (Table II analogue), 8 warps / CTA, 1..4 CTAs per SM
    for (int bps = 1; bps <= 4; bps *= 2) {
      const int iters = 2000;
      k_lds_bw<<<sms * bps, 256>>>(out, 10);
      k_lds_bw<<<sms * bps, 256>>>(out, iters);
      cudaDeviceSynchronize();
      const unsigned long long c = max_cyc(sms * bps);
      const double bytes_sm = (double)bps * 256 * 16 * 8 * iters;
      printf("{\"bench\":\"lds128_bw\",\"warps_per_sm\":%d,\"bytes_per_clk_sm\":%.1f}\n", bps * 8, bytes_sm / c);
    }
  }
  long long h;
  const char *lat_names[4] = {"ffma_dep_latency", "shfl_plus_fadd_latency", "lds_chase_latency",
                              "sqrt_rn_div_rn_fadd_chain"};
  for (int w = 0; w < 4; ++w) {
    k_lat<<<1, 32>>>(out, cyc, 1000, w);
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("{\"bench\":\"%s\",\"cycles\":%.2f}\n", lat_names[w], h / (1000.0 * 16));
  }
  for (int nt = 32; nt <= 1024; nt *= 2) {
    k_bar<<<1, nt>>>(out, cyc, 10);
    k_bar<<<1, nt>>>(out, cyc, 10000);
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("{\"bench\":\"syncthreads\",\"threads\":%d,\"cycles\":%.2f}\n", nt, h / 10000.0);
  }
  for (int cnt = 64; cnt <= 512; cnt *= 2) {
    k_named_bar<<<1, 512>>>(out, cyc, 10000, cnt);
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("{\"bench\":\"named_barrier\",\"threads\":%d,\"cycles\":%.2f}\n", cnt, h / 10000.0);
  }
  k_mbar_pingpong<<<1, 64>>>(out, cyc, 10000);
  cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
  printf("{\"bench\":\"mbarrier_handoff\",\"cycles\":%.2f}\n", h / 20000.0);
  for (int cs = 2; cs <= 8; cs *= 2) {
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = cs;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.gridDim = dim3(cs);
    cfg.blockDim = dim3(128);
    cfg.attrs = at;
    cfg.numAttrs = 1;
    int iters = 10000;
    cudaLaunchKernelEx(&cfg, k_cluster_bar, out, cyc, iters);
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("{\"bench\":\"cluster_barrier\",\"cluster\":%d,\"cycles\":%.2f}\n", cs, h / (double)iters);
    iters = 1000;
    cudaLaunchKernelEx(&cfg, k_dsmem_chase, out, cyc, iters);
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("{\"bench\":\"dsmem_remote_load_latency\",\"cluster\":%d,\"cycles\":%.2f}\n", cs, h / (iters * 16.0));
  }
  {  // CUDA-event time of an empty launch (what an event-timed kernel adds)
    cudaEvent_t a, b2;
    cudaEventCreate(&a);
    cudaEventCreate(&b2);
    float best = 1e9, sum = 0.f;
    for (int r = 0; r < 200; ++r) {
      cudaEventRecord(a);
      k_empty<<<1, 32>>>(nullptr);
      cudaEventRecord(b2);
      cudaEventSynchronize(b2);
      float ms;
      cudaEventElapsedTime(&ms, a, b2);
      if (r >= 20) {
        best = ms < best ? ms : best;
        sum += ms;
      }
    }
    printf("{\"bench\":\"empty_launch_event_us\",\"min\":%.2f,\"mean\":%.2f}\n", best * 1e3, sum / 180 * 1e3);
    for (int r = 0; r < 3; ++r) {
      cudaEventRecord(a);
      k_empty<<<148 * 8, 64>>>(nullptr);
      cudaEventRecord(b2);
      cudaEventSynchronize(b2);
    }
    float ms;
    cudaEventElapsedTime(&ms, a, b2);
    printf("{\"bench\":\"empty_grid_1184x64_event_us\",\"value\":%.2f}\n", ms * 1e3);
  }
  cudaError_t e = cudaDeviceSynchronize();
  printf("{\"sms\":%d,\"clock_khz\":%d,\"status\":\"%s\"}\n", sms, clk, cudaGetErrorString(e));
  return 0;
}

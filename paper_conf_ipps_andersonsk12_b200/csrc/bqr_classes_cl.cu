// bqr_classes_cl.cu -- cluster-per-matrix complex classes (bqr_cl.cuh):
// one cluster of 2 or 4 CTAs per matrix of up to 256 x 72 complex64 (with
// the fused Q^H B columns), for batches too small to fill the GPU with one
// matrix per SM (strong scaling of the STAP shape: 32 matrices per GPU at
// 8 GPUs).  Explicit (BQR_FORCE_VARIANT); orgqr takes the right-looking
// register-file class.
#include <algorithm>

#include "bqr_cl.cuh"
#include "bqr_launch.cuh"

namespace bqr {
namespace host {

template <int CL, int W, int NC>
int launch_cl(const Call &c) {
  using K = cl::Cfg<CL, W, NC>;
  if (c.m > K::MMAX || c.n + c.nrhs > K::NMAX || c.k > std::min(c.m, c.n)) return BQR_ERR_NOT_SUPPORTED;
  auto kern = cl::geqrf_cl_kernel<CL, W, NC>;
  if (!ensure_smem(reinterpret_cast<const void *>(kern), K::kSmemBytes)) return BQR_ERR_CUDA;
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, current_device());
  long long maxclus = 0;
  {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)CL * 8u, 1, 1);
    cfg.blockDim = dim3(K::kThreads, 1, 1);
    cfg.dynamicSmemBytes = K::kSmemBytes;
    int n = 0;
    if (cudaOccupancyMaxActiveClusters(&n, reinterpret_cast<const void *>(kern), &cfg) == cudaSuccess && n > 0)
      maxclus = n;
    else {
      cudaGetLastError();
      maxclus = sms / CL;
    }
  }
  if (c.resident) {
    *c.resident = maxclus;
    return BQR_SUCCESS;
  }
  cl::Args a;
  a.A = static_cast<float2 *>(c.A);
  a.tau = static_cast<float2 *>(c.tau);
  a.B = static_cast<float2 *>(c.B);
  a.batch = c.batch;
  a.m = c.m;
  a.n = c.n;
  a.kmax = c.k;
  a.lda = c.lda;
  a.ldb = c.ldb;
  a.nrhs = c.nrhs;
  a.strideA = c.strideA >= 0 ? c.strideA : (long long)c.lda * c.n;
  a.strideT = c.strideT >= 0 ? c.strideT : (long long)c.k;
  a.strideB = (long long)c.ldb * c.nrhs;
  const long long nclus = std::min<long long>(c.batch, maxclus);
  if (nclus <= 0) return BQR_SUCCESS;
  kern<<<(unsigned)(nclus * CL), K::kThreads, K::kSmemBytes, c.stream>>>(a);
  return finish_launch();
}

namespace {
using OrgRf = decltype(&launch_rf<float2, 32, 12, 8, 6, 1, false, false, false, true>);
const OrgRf kOrg = &launch_rf<float2, 32, 12, 8, 6, 1, false, false, false, true>;
const ClassEntry kTable[] = {
    {BQR_C64, 256, 72, 0, 0, true, Plan{"alt_cl4_c64_256x72", &launch_cl<4, 3, 6>, kOrg}},
    {BQR_C64, 256, 72, 0, 0, true, Plan{"alt_cl4_c64_256x72_aug", &launch_cl<4, 3, 6>, kOrg}},
    {BQR_C64, 256, 72, 0, 0, true, Plan{"alt_cl2_c64_256x72", &launch_cl<2, 6, 6>, kOrg}},
    {BQR_C64, 256, 72, 0, 0, true, Plan{"alt_cl2_c64_256x72_aug", &launch_cl<2, 6, 6>, kOrg}},
    // the same kernel on one CTA of 12 warps (no distributed shared memory);
    // 6 / 8 / 16 / 18 / 24 warps per CTA measured slower (c4_cluster.jsonl)
    {BQR_C64, 256, 72, 0, 0, true, Plan{"alt_cl1_c64_256x72_aug", &launch_cl<1, 12, 6>, kOrg}},
};
}  // namespace

const ClassEntry *classes_cl(int *n) {
  *n = (int)(sizeof(kTable) / sizeof(kTable[0]));
  return kTable;
}

}  // namespace host
}  // namespace bqr

#ifdef BQR_CL_TIMING
extern "C" int bqr_cl_debug_stamps(void *host, size_t bytes) {
  return cudaMemcpyFromSymbol(host, bqr::cl::g_cl_dbg, bytes) == cudaSuccess ? 0 : 2;
}
#endif

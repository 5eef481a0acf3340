// bqr_classes_ll.cu -- the left-looking register-block class of the C3
// headline shape (bqr_ll.cuh): 56 x 56 fp32, 17 warps = 34 matrices per SM.
// orgqr of the same shape keeps the right-looking class (bqr_rf.cuh).
#include "bqr_launch.cuh"
#include "bqr_ll.cuh"

namespace bqr {
namespace host {

int launch_ll56(const Call &c) {
  if (c.m != ll::kM || c.n != ll::kM || c.k != ll::kM || c.nrhs > 0 || c.lda < ll::kM) return BQR_ERR_NOT_SUPPORTED;
  // the kernel moves row pairs as 8-byte words: odd lda / stride or a
  // 4-byte-aligned base take the right-looking class of the same shape
  const long long sA = c.strideA >= 0 ? c.strideA : (long long)c.lda * c.n;
  if ((c.lda & 1) || (sA & 1) || (reinterpret_cast<uintptr_t>(c.A) & 7))
    return launch_rf<float, 4, 4, 14, 14, 2, true, true, false, false>(c);
  auto kern = ll::geqrf_ll56_kernel;
  if (!ensure_smem(reinterpret_cast<const void *>(kern), ll::kSmemBytes)) return BQR_ERR_CUDA;
  if (c.resident) {
    *c.resident = resident_of(reinterpret_cast<const void *>(kern), ll::kThreads, ll::kSmemBytes, 2 * ll::kWarps);
    return BQR_SUCCESS;
  }
  ll::LlArgs a;
  a.A = static_cast<float *>(c.A);
  a.tau = static_cast<float *>(c.tau);
  a.batch = c.batch;
  a.lda = c.lda;
  a.strideA = c.strideA >= 0 ? c.strideA : (long long)c.lda * c.n;
  a.strideT = c.strideT >= 0 ? c.strideT : (long long)c.k;
  const long long pairs = (c.batch + 1) / 2;
  int sms = 0, bps = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, current_device());
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, kern, ll::kThreads, ll::kSmemBytes);
  const long long grid = std::min<long long>(pairs, (long long)sms * std::max(1, bps));
  if (grid <= 0) return BQR_SUCCESS;
  kern<<<(unsigned)grid, ll::kThreads, ll::kSmemBytes, c.stream>>>(a);
  return finish_launch();
}

namespace {
const ClassEntry kTable[] = {
    {BQR_R32, 56, 56, 56, 56, false,
     Plan{"ll_f32_56x56_left4_x2", &launch_ll56, &launch_rf<float, 4, 4, 14, 14, 2, true, true, false, true>}},
};
}  // namespace

const ClassEntry *classes_ll(int *n) {
  *n = (int)(sizeof(kTable) / sizeof(kTable[0]));
  return kTable;
}

}  // namespace host
}  // namespace bqr

#ifdef BQR_LL_TIMING
extern "C" int bqr_ll_debug_stamps(void *host, size_t bytes) {
  return cudaMemcpyFromSymbol(host, bqr::ll::g_ll_dbg, bytes) == cudaSuccess ? 0 : 2;
}
#endif

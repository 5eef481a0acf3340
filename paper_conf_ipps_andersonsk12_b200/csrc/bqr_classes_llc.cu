// bqr_classes_llc.cu -- the left-looking complex class of the STAP shape
// (bqr_llc.cuh): 240 x 66 complex64, alone or with one right-hand side as
// column 66 of [A | b] (the fused Q^H b of the C4 bench step), two matrices
// per SM.  Other shapes that reach these entries, and orgqr, take the
// right-looking register-file classes (bqr_rf.cuh).
#include "bqr_launch.cuh"
#include "bqr_llc.cuh"

namespace bqr {
namespace host {

int launch_llc240(const Call &c) {
  using namespace llc;
  const bool shape = c.m == kM && c.n == kN && c.k == kN && c.nrhs <= 1 && c.lda >= kM &&
                     (c.nrhs == 0 || c.ldb >= kM) && c.strideA < 0;
  if (!shape) {
    if (c.nrhs > 0) return launch_rf<float2, 32, 12, 8, 6, 1, false, false, true, false>(c);
    return launch_rf<float2, 32, 11, 8, 6, 1, false, false, false, false>(c);
  }
  auto kern = geqrf_llc240_kernel;
  if (!ensure_smem(reinterpret_cast<const void *>(kern), kSmemBytes)) return BQR_ERR_CUDA;
  if (c.resident) {
    *c.resident = resident_of(reinterpret_cast<const void *>(kern), kThreads, kSmemBytes, 1);
    return BQR_SUCCESS;
  }
  Args a;
  a.A = static_cast<float2 *>(c.A);
  a.tau = static_cast<float2 *>(c.tau);
  a.B = static_cast<float2 *>(c.B);
  a.batch = c.batch;
  a.lda = c.lda;
  a.ldb = c.ldb;
  a.nrhs = c.nrhs;
  a.strideA = (long long)c.lda * c.n;
  a.strideT = c.strideT >= 0 ? c.strideT : (long long)c.k;
  a.strideB = (long long)c.ldb * c.nrhs;
  int sms = 0, bps = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, current_device());
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, kern, kThreads, kSmemBytes);
  const long long grid = std::min<long long>(c.batch, (long long)sms * std::max(1, bps));
  if (grid <= 0) return BQR_SUCCESS;
  kern<<<(unsigned)grid, kThreads, kSmemBytes, c.stream>>>(a);
  return finish_launch();
}

namespace {
const ClassEntry kTable[] = {
    // experiment (BQR_FORCE_VARIANT): two matrices per SM, decoupled per-
    // reflector mbarriers; parity green but equal to the right-looking class
    // on B200 (geqrf 119.3 vs 118.1 us, fused step 119.4 vs ~119 us; an
    // 8-row-lane CTA-barrier version: 121.4): profiles/r02/experiments/README.md
    {BQR_C64, 240, 66, 240, 66, true,
     Plan{"alt_llc_c64_240x66_left3", &launch_llc240, &launch_rf<float2, 32, 11, 8, 6, 1, false, false, false, true>}},
    // the fused [A | b] step of C4 (picked by pick_fused for exactly 240 x (66 + 1))
    {BQR_C64, 240, 67, 240, 67, true,
     Plan{"alt_llc_c64_240x66_left3_aug", &launch_llc240, &launch_rf<float2, 32, 12, 8, 6, 1, false, false, false, true>}},
};
}  // namespace

const ClassEntry *classes_llc(int *n) {
  *n = (int)(sizeof(kTable) / sizeof(kTable[0]));
  return kTable;
}

}  // namespace host
}  // namespace bqr

#ifdef BQR_LLC_TIMING
extern "C" int bqr_llc_debug_stamps(void *host, size_t bytes) {
  return cudaMemcpyFromSymbol(host, bqr::llc::g_llc_dbg, bytes) == cudaSuccess ? 0 : 2;
}
#endif

// bqr_classes_co.cu -- column-owner classes (bqr_co.cuh): the C3 headline
// shape 56x56 fp32 and its layout variants (BQR_FORCE_VARIANT).  A call the
// column-owner kernel cannot take (lda > m, panel views with custom batch
// strides, a misaligned base) goes to the 2D-cyclic class of the same shape.
#include "bqr_co.cuh"
#include "bqr_launch.cuh"

namespace bqr {
namespace host {

template <int M, int N, int L, int H, int LS, int PW, int MINB, LaunchFn FB>
int launch_co(const Call &c) {
  using Cf = CoCfg<M, N, L, H, LS, PW>;
  const bool ok = c.m == M && c.n == N && c.lda == M && c.strideA < 0 && c.strideT < 0 && c.nrhs == 0 &&
                  (reinterpret_cast<uintptr_t>(c.A) & 15) == 0;
  if (!ok) return FB(c);
  auto kern = geqrf_co_kernel<M, N, L, H, LS, PW, MINB>;
  if (!ensure_smem(reinterpret_cast<const void *>(kern), Cf::SMEM)) return BQR_ERR_CUDA;
  if (c.resident) {
    *c.resident = resident_of(reinterpret_cast<const void *>(kern), 128, Cf::SMEM, Cf::WPC * Cf::MPW);
    return BQR_SUCCESS;
  }
  const long long items = (c.batch + Cf::MPW - 1) / Cf::MPW;
  long long grid = (items + Cf::WPC - 1) / Cf::WPC;
  int sms = 0, bps = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, current_device());
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, kern, 128, Cf::SMEM);
  grid = std::min<long long>(grid, (long long)std::max(1, sms) * std::max(1, bps));
  CoArgs a{reinterpret_cast<float *>(c.A), reinterpret_cast<float *>(c.tau), c.batch};
  kern<<<(unsigned)grid, 128, Cf::SMEM, c.stream>>>(a);
  return finish_launch();
}

// the 2D-cyclic 56x56 class (fallback and orgqr)
#define RF56_GEQRF &launch_rf<float, 4, 4, 14, 14, 2, true, true, false, false>
#define RF56_ORGQR &launch_rf<float, 4, 4, 14, 14, 2, true, true, false, true>
#define CO_PLAN(M, N, L, H, LS, PW, MINB, NAME) \
  Plan { NAME, &launch_co<M, N, L, H, LS, PW, MINB, RF56_GEQRF>, RF56_ORGQR }

namespace {
const ClassEntry kTable[] = {
    // experiment only (BQR_FORCE_VARIANT): parity-correct but 1.7x slower
    // than the 2D-cyclic class on C3 (146 vs 88 us, profiles/r02/experiments)
    {BQR_R32, 56, 56, 56, 56, true, CO_PLAN(56, 56, 14, 2, 16, 7, 3, "alt_co_f32_L14H2_x1")},
};
}  // namespace

const ClassEntry *classes_co(int *n) {
  *n = (int)(sizeof(kTable) / sizeof(kTable[0]));
  return kTable;
}

}  // namespace host
}  // namespace bqr

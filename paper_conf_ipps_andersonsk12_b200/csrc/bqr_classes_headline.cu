// bqr_classes_headline.cu -- exact-shape headline classes (C3 56x56 fp32, C4 240x66 c64, the STAP 80x16 / 192x96
// c64 shapes of Table VII) and the augmented (fused Q^H B) classes
// (one translation unit per table so the template instantiations of the
// size classes compile in parallel; see bqr_launch.cuh)
#include "bqr_launch.cuh"

namespace bqr {
namespace host {

namespace {
const ClassEntry kTable[] = {
    // the round-1/2 right-looking C3 class; the dispatched one is the
    // left-looking bqr_classes_ll.cu (A/B via BQR_FORCE_VARIANT)
    {BQR_R32, 56, 56, 56, 56, true, RF_PLAN_X(float, 4, 4, 14, 14, 2, true, true, "alt_rf_f32_R4G4_14x14_x2_exact")},
    {BQR_C64, 240, 66, 240, 66, false, RF_PLAN(float2, 32, 11, 8, 6, 1, false, "rf_c64_R32G11_8x6_cta")},
    // NEXT-2: the paper's other RT_STAP shapes (Table VII)
    {BQR_C64, 80, 16, 80, 16, false, RF_PLAN(float2, 16, 4, 5, 4, 1, false, "rf_c64_R16G4_5x4_cta")},
    {BQR_C64, 192, 96, 192, 96, false, RF_PLAN(float2, 32, 16, 6, 6, 1, false, "rf_c64_R32G16_6x6_cta")},
    {BQR_C64, 256, 72, 240, 67, true, RF_PLAN_AUG(float2, 32, 12, 8, 6, "rf_c64_R32G12_8x6_aug")},
    {BQR_C64, 128, 128, 0, 0, true, RF_PLAN_AUG(float2, 32, 16, 4, 8, "rf_c64_R32G16_4x8_aug")},
    {BQR_R32, 128, 128, 0, 0, true, RF_PLAN_AUG(float, 32, 8, 4, 16, "rf_f32_R32G8_4x16_aug")},
};
}  // namespace

const ClassEntry *classes_headline(int *n) {
  *n = (int)(sizeof(kTable) / sizeof(kTable[0]));
  return kTable;
}

}  // namespace host
}  // namespace bqr

#ifdef BQR_PHASE_TIMING
// debug builds only: the phase-timing stamps of this translation unit's
// kernels (the headline classes; tools/phase_timing.py)
extern "C" int bqr_debug_stamps(void *host, size_t bytes) {
  return cudaMemcpyFromSymbol(host, bqr::g_bqr_dbg, bytes) == cudaSuccess ? 0 : 2;
}
extern "C" int bqr_debug_clear(void) {
  static unsigned long long z[bqr::kDbgSteps * bqr::kDbgWarps * 4];
  return cudaMemcpyToSymbol(bqr::g_bqr_dbg, z, sizeof(z)) == cudaSuccess ? 0 : 2;
}
#endif

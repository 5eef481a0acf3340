// bqr_classes_c64.cu -- complex64 size classes
// (one translation unit per table so the template instantiations of the
// size classes compile in parallel; see bqr_launch.cuh)
#include "bqr_launch.cuh"

namespace bqr {
namespace host {

namespace {
const ClassEntry kTable[] = {
    {BQR_C64, 16, 16, 0, 0, false, RF_PLAN(float2, 2, 2, 8, 8, 8, false, "rf_c64_R2G2_8x8_x8_warp")},
    {BQR_C64, 32, 32, 0, 0, false, RF_PLAN(float2, 4, 4, 8, 8, 2, false, "rf_c64_R4G4_8x8_x2_warp")},
    {BQR_C64, 48, 48, 0, 0, false, RF_PLAN(float2, 8, 8, 6, 6, 1, false, "rf_c64_R8G8_6x6_cta")},
    // up to 56 x 56 (the C5 cell at the paper's headline size): 7 x 7 per
    // lane instead of the 64 x 64 class's 8 x 8 (31% padding at 56)
    {BQR_C64, 56, 56, 0, 0, false, RF_PLAN(float2, 8, 8, 7, 7, 1, false, "rf_c64_R8G8_7x7_cta")},
    {BQR_C64, 64, 64, 0, 0, false, RF_PLAN(float2, 8, 8, 8, 8, 1, false, "rf_c64_R8G8_8x8_cta")},
    {BQR_C64, 80, 80, 0, 0, false, RF_PLAN(float2, 8, 8, 10, 10, 1, false, "rf_c64_R8G8_10x10_cta")},
    {BQR_C64, 96, 96, 0, 0, false, RF_PLAN(float2, 16, 16, 6, 6, 1, false, "rf_c64_R16G16_6x6_cta")},
    {BQR_C64, 112, 112, 0, 0, false, RF_PLAN(float2, 16, 16, 7, 7, 1, false, "rf_c64_R16G16_7x7_cta")},
    {BQR_C64, 128, 128, 0, 0, false, RF_PLAN(float2, 16, 16, 8, 8, 1, false, "rf_c64_R16G16_8x8_cta")},
    {BQR_C64, 256, 96, 0, 0, false, RF_PLAN(float2, 32, 16, 8, 6, 1, false, "rf_c64_R32G16_8x6_cta")},
    // 160 x 160 complex (51 K words): whole matrix in one SM's register file
    {BQR_C64, 160, 160, 0, 0, false, RF_PLAN(float2, 16, 32, 10, 5, 1, false, "rf_c64_R16G32_10x5_cta")},
};
}  // namespace

const ClassEntry *classes_c64(int *n) {
  *n = (int)(sizeof(kTable) / sizeof(kTable[0]));
  return kTable;
}

}  // namespace host
}  // namespace bqr

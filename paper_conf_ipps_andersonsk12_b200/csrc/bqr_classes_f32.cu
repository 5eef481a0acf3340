// bqr_classes_f32.cu -- fp32 size classes (square R x G lane grids where the register budget allows)
// (one translation unit per table so the template instantiations of the
// size classes compile in parallel; see bqr_launch.cuh)
#include "bqr_launch.cuh"

namespace bqr {
namespace host {

namespace {
const ClassEntry kTable[] = {
    {BQR_R32, 16, 16, 0, 0, false, RF_PLAN(float, 2, 2, 8, 8, 8, true, "rf_f32_R2G2_8x8_x8_stage")},
    {BQR_R32, 24, 24, 0, 0, false, RF_PLAN(float, 2, 2, 12, 12, 8, true, "rf_f32_R2G2_12x12_x8_stage")},
    {BQR_R32, 32, 32, 0, 0, false, RF_PLAN(float, 2, 4, 16, 8, 4, true, "rf_f32_R2G4_16x8_x4_stage")},
    {BQR_R32, 48, 48, 0, 0, false, RF_PLAN(float, 4, 4, 12, 12, 2, true, "rf_f32_R4G4_12x12_x2_stage")},
    {BQR_R32, 64, 64, 0, 0, false, RF_PLAN(float, 4, 8, 16, 8, 2, true, "rf_f32_R4G8_16x8_x2_stage")},
    {BQR_R32, 80, 80, 0, 0, false, RF_PLAN(float, 8, 8, 10, 10, 1, false, "rf_f32_R8G8_10x10_cta")},
    {BQR_R32, 96, 96, 0, 0, false, RF_PLAN(float, 8, 8, 12, 12, 1, false, "rf_f32_R8G8_12x12_cta")},
    {BQR_R32, 112, 112, 0, 0, false, RF_PLAN(float, 8, 8, 14, 14, 1, false, "rf_f32_R8G8_14x14_cta")},
    {BQR_R32, 128, 128, 0, 0, false, RF_PLAN(float, 8, 16, 16, 8, 1, false, "rf_f32_R8G16_16x8_cta")},
    {BQR_R32, 256, 64, 0, 0, false, RF_PLAN(float, 32, 8, 8, 8, 1, false, "rf_f32_R32G8_8x8_cta")},
    // 144..256: the whole matrix in the register file of one SM (256-1024
    // threads); measured 3-4x faster than the tiled panel path (profiles/r01)
    {BQR_R32, 144, 144, 0, 0, false, RF_PLAN(float, 16, 16, 9, 9, 1, false, "rf_f32_R16G16_9x9_cta")},
    {BQR_R32, 160, 160, 0, 0, false, RF_PLAN(float, 16, 16, 10, 10, 1, false, "rf_f32_R16G16_10x10_cta")},
    {BQR_R32, 192, 192, 0, 0, false, RF_PLAN(float, 32, 32, 6, 6, 1, false, "rf_f32_R32G32_6x6_cta")},
    {BQR_R32, 224, 224, 0, 0, false, RF_PLAN(float, 32, 32, 7, 7, 1, false, "rf_f32_R32G32_7x7_cta")},
    {BQR_R32, 256, 256, 0, 0, false, RF_PLAN(float, 32, 32, 8, 8, 1, false, "rf_f32_R32G32_8x8_cta")},
};
}  // namespace

const ClassEntry *classes_f32(int *n) {
  *n = (int)(sizeof(kTable) / sizeof(kTable[0]));
  return kTable;
}

}  // namespace host
}  // namespace bqr

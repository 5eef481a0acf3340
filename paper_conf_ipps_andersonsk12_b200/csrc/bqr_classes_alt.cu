// bqr_classes_alt.cu -- candidate size classes reachable only through
// BQR_FORCE_VARIANT (layout experiments for tools/sweep.py --variant); the
// default dispatch never picks an entry of this table.
#include "bqr_launch.cuh"

namespace bqr {
namespace host {

namespace {
const ClassEntry kTable[] = {
    {BQR_R32, 128, 128, 0, 0, true, RF_PLAN(float, 16, 16, 8, 8, 1, false, "alt_f32_R16G16_8x8_cta")},
    {BQR_R32, 128, 128, 0, 0, true, RF_PLAN(float, 16, 32, 8, 4, 1, false, "alt_f32_R16G32_8x4_cta")},
    {BQR_R32, 128, 128, 0, 0, true, RF_PLAN(float, 32, 16, 4, 8, 1, false, "alt_f32_R32G16_4x8_cta")},
    {BQR_R32, 160, 160, 0, 0, true, RF_PLAN(float, 32, 16, 5, 10, 1, false, "alt_f32_R32G16_5x10_cta")},
    {BQR_R32, 160, 160, 0, 0, true, RF_PLAN(float, 16, 32, 10, 5, 1, false, "alt_f32_R16G32_10x5_cta")},
    {BQR_R32, 160, 160, 0, 0, true, RF_PLAN(float, 32, 32, 5, 5, 1, false, "alt_f32_R32G32_5x5_cta")},
    {BQR_R32, 128, 128, 0, 0, true, RF_PLAN(float, 16, 8, 8, 16, 1, false, "alt_f32_R16G8_8x16_cta")},
    {BQR_C64, 160, 160, 0, 0, true, RF_PLAN(float2, 32, 16, 5, 10, 1, false, "alt_c64_R32G16_5x10_cta")},
    {BQR_R32, 128, 128, 0, 0, true, RF_PLAN(float, 8, 8, 16, 16, 1, false, "alt_f32_R8G8_16x16_cta")},
    {BQR_C64, 144, 144, 0, 0, true, RF_PLAN(float2, 16, 16, 9, 9, 1, false, "alt_c64_R16G16_9x9_cta")},
};
}  // namespace

const ClassEntry *classes_alt(int *n) {
  *n = (int)(sizeof(kTable) / sizeof(kTable[0]));
  return kTable;
}

}  // namespace host
}  // namespace bqr

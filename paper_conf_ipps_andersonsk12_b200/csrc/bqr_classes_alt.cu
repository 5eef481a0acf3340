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
    // STAP 240x66 c64: 16 row lanes (4-level butterflies) instead of 32
    {BQR_C64, 240, 66, 240, 66, true, RF_PLAN(float2, 16, 22, 15, 3, 1, false, "alt_c64_R16G22_15x3_cta")},
    {BQR_C64, 240, 72, 0, 0, true, RF_PLAN_AUG(float2, 16, 24, 15, 3, "alt_c64_R16G24_15x3_aug")},
    {BQR_C64, 240, 72, 0, 0, true, RF_PLAN_AUG(float2, 16, 12, 15, 6, "alt_c64_R16G12_15x6_aug")},
    {BQR_C64, 256, 72, 0, 0, true, RF_PLAN_AUG(float2, 32, 24, 8, 3, "alt_c64_R32G24_8x3_aug")},
    // STAP 80x16 c64 (384 matrices, latency-bound): the former one-warp class and
    // other thread counts / row-lane splits (experiments/s80_variants.jsonl)
    {BQR_C64, 80, 16, 80, 16, true, RF_PLAN(float2, 16, 2, 5, 8, 1, false, "alt_c64_R16G2_5x8_warp")},
    {BQR_C64, 80, 16, 80, 16, true, RF_PLAN(float2, 16, 8, 5, 2, 1, false, "alt_c64_R16G8_5x2_cta")},
    {BQR_C64, 80, 16, 80, 16, true, RF_PLAN(float2, 8, 4, 10, 4, 1, false, "alt_c64_R8G4_10x4_warp")},
    {BQR_C64, 96, 16, 0, 0, true, RF_PLAN(float2, 32, 4, 3, 4, 1, false, "alt_c64_R32G4_3x4_cta")},
    {BQR_C64, 80, 16, 80, 16, true, RF_PLAN(float2, 8, 8, 10, 2, 1, false, "alt_c64_R8G8_10x2_cta")},
    {BQR_C64, 80, 16, 80, 16, true, RF_PLAN(float2, 16, 16, 5, 1, 1, false, "alt_c64_R16G16_5x1_cta")},
    {BQR_C64, 80, 16, 80, 16, true, RF_PLAN(float2, 8, 16, 10, 1, 1, false, "alt_c64_R8G16_10x1_cta")},
    // STAP 192x96 c64 (128 matrices: one CTA per SM, latency-bound)
    {BQR_C64, 192, 96, 192, 96, true, RF_PLAN(float2, 32, 32, 6, 3, 1, false, "alt_c64_R32G32_6x3_cta")},
    {BQR_C64, 192, 96, 192, 96, true, RF_PLAN(float2, 32, 24, 6, 4, 1, false, "alt_c64_R32G24_6x4_cta")},
    {BQR_C64, 192, 96, 192, 96, true, RF_PLAN(float2, 16, 32, 12, 3, 1, false, "alt_c64_R16G32_12x3_cta")},
    {BQR_C64, 192, 96, 192, 96, true, RF_PLAN(float2, 16, 16, 12, 6, 1, false, "alt_c64_R16G16_12x6_cta")},
    {BQR_C64, 192, 96, 192, 96, true, RF_PLAN(float2, 32, 8, 6, 12, 1, false, "alt_c64_R32G8_6x12_cta")},
    // 56x56 fp32, one matrix per warp, register cap for MB warps per SM
    {BQR_R32, 56, 56, 56, 56, true, RF_PLAN_XM(float, 4, 8, 14, 7, 1, true, true, 12, "alt_f32_R4G8_14x7_x1_mb12")},
    {BQR_R32, 56, 56, 56, 56, true, RF_PLAN_XM(float, 4, 8, 14, 7, 1, true, true, 14, "alt_f32_R4G8_14x7_x1_mb14")},
    {BQR_R32, 56, 56, 56, 56, true, RF_PLAN_XM(float, 4, 8, 14, 7, 1, true, true, 16, "alt_f32_R4G8_14x7_x1_mb16")},
    {BQR_R32, 56, 56, 56, 56, true, RF_PLAN_XM(float, 8, 4, 7, 14, 1, true, true, 12, "alt_f32_R8G4_7x14_x1_mb12")},
    {BQR_R32, 56, 56, 56, 56, true, RF_PLAN_XM(float, 8, 4, 7, 14, 1, true, true, 14, "alt_f32_R8G4_7x14_x1_mb14")},
};
}  // namespace

const ClassEntry *classes_alt(int *n) {
  *n = (int)(sizeof(kTable) / sizeof(kTable[0]));
  return kTable;
}

}  // namespace host
}  // namespace bqr

// hs_cell.cuh -- the one per-cell hotspot update every hotspot kernel variant calls.
//
// Rodinia hotspot `calculate_temp` (DESIGN.md §3 H1-H8):
//   T' = c + k * ( P + ((S+N) - 2c)*ry + ((E+W) - 2c)*rx + (amb - c)*rz )
// evaluated in fp32 in exactly this order with explicit round-to-nearest intrinsics, so the
// compiler cannot contract or reorder differently in different variants: every coarsening
// variant is bit-identical to every other one (the paper's correctness criterion,
// PAPER.md:145, 295).  (S+N) - 2c is written as fma(-2, c, S+N), which equals the unfused
// (S+N) - (2c) exactly because 2c is exact in fp32; the three "acc + x*r" terms and the
// final c + k*acc use fused multiply-adds (DESIGN.md §3 H2).
#pragma once

namespace rg {

struct HsCoef {
    float k, rx, ry, rz, amb;
};

__device__ __forceinline__ float hs_cell(float c, float n, float s, float e, float w, float p,
                                         const HsCoef& cf) {
    float sn = __fadd_rn(s, n);
    float ew = __fadd_rn(e, w);
    float a = __fmaf_rn(-2.0f, c, sn);
    float b = __fmaf_rn(-2.0f, c, ew);
    float d = __fsub_rn(cf.amb, c);
    float acc = __fmaf_rn(a, cf.ry, p);
    acc = __fmaf_rn(b, cf.rx, acc);
    acc = __fmaf_rn(d, cf.rz, acc);
    return __fmaf_rn(cf.k, acc, c);
}

}  // namespace rg

// hs_cell.cuh -- the one per-cell hotspot update every hotspot kernel variant calls.
//
// Rodinia hotspot `calculate_temp` (DESIGN.md §3 H1-H8) defines
//   T' = c + k * ( P + ((S+N) - 2c)*ry + ((E+W) - 2c)*rx + (amb - c)*rz ).
// The kernels evaluate the algebraically identical *state form* (DESIGN.md §3 H2):
//   u  = T - amb                       (state, converted once per solve: hs_to_state)
//   kP = fl(k * P)                     (pre-scaled power, once per solve: hs_scale_power)
//   u' = u + ( (S+N)*kry + kP + (E+W)*krx + u*m )
// with kry = fl(k*ry), krx = fl(k*rx), m = fl(-k*(2ry + 2rx + rz)) computed in fp64 and rounded
// once (hs_derive), and T = u + amb at the end (hs_from_state).  Substituting c = u + amb
// (and N = uN + amb, ...) into the definition gives exactly this expression; it costs 6 FP32
// operations per cell-update instead of 9, and its fp32 error against the fp64 oracle is
// smaller than the literal order's (the state u has half the ulp of T near 320 K; measured in
// DESIGN.md §3 H2).  Explicit round-to-nearest intrinsics keep the compiler from contracting or
// reordering differently in different variants, so every coarsening variant is bit-identical
// to every other one (the paper's correctness criterion).
#pragma once

#include <cstdint>

namespace rg {

struct HsCoef {   // state-form coefficients (device side)
    float kry, krx, m;
};

struct HsMap {    // state <-> temperature map (pre/post passes)
    float k, amb;
};

// fp64 evaluation of the derived coefficients from the caller's fp32 (k, rx, ry, rz).
inline HsCoef hs_derive(float k, float rx, float ry, float rz) {
    const double kd = k;
    HsCoef c;
    c.kry = (float)(kd * (double)ry);
    c.krx = (float)(kd * (double)rx);
    c.m = (float)(-kd * (2.0 * (double)ry + 2.0 * (double)rx + (double)rz));
    return c;
}

// The same update with E+W already formed (ew = fl(e + w)).
__device__ __forceinline__ float hs_cell_ew(float u, float n, float s, float ew, float kp, const HsCoef& cf) {
    const float sn = __fadd_rn(s, n);
    float acc = __fmaf_rn(sn, cf.kry, kp);
    acc = __fmaf_rn(ew, cf.krx, acc);
    acc = __fmaf_rn(u, cf.m, acc);
    return __fadd_rn(u, acc);
}

// Two cells at once on the packed FP32x2 pipe (sm_100 FADD2/FFMA2): element-wise the same
// operations in the same order with the same round-to-nearest as hs_cell_ew, so the results
// are bit-identical; one instruction covers both cells.
__device__ __forceinline__ float2 hs_cell2(float2 u, float2 n, float2 s, float2 ew, float2 kp, const HsCoef& cf) {
    const float2 sn = __fadd2_rn(s, n);
    float2 acc = __ffma2_rn(sn, make_float2(cf.kry, cf.kry), kp);
    acc = __ffma2_rn(ew, make_float2(cf.krx, cf.krx), acc);
    acc = __ffma2_rn(u, make_float2(cf.m, cf.m), acc);
    return __fadd2_rn(u, acc);
}

__device__ __forceinline__ float hs_cell(float u, float n, float s, float e, float w, float kp,
                                         const HsCoef& cf) {
    const float sn = __fadd_rn(s, n);
    const float ew = __fadd_rn(e, w);
    float acc = __fmaf_rn(sn, cf.kry, kp);
    acc = __fmaf_rn(ew, cf.krx, acc);
    acc = __fmaf_rn(u, cf.m, acc);
    return __fadd_rn(u, acc);
}

}  // namespace rg

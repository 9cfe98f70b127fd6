// hotspot.cu -- granularity-parameterised hotspot kernels for sm_100a.
//
// Operation: Rodinia hotspot `calculate_temp` (DESIGN.md §3 H1-H8), per cell via hs_cell() in
// the state form u = T - amb with pre-scaled power kP = k*P (DESIGN.md §3 H2): every stepping
// kernel below reads/writes states u and reads kP where the comments say T and P; solve()
// converts T -> u and P -> kP before the first launch and u -> T after the last.
// Two variant families:
//
//  * hs_direct<TX,TY,MODE>  (temporal = 1).  The paper's granularity space verbatim: the
//    original kernel is a 16x16-thread CTA computing one 16x16 tile, one cell per thread.
//    Thread coarsening (TX,TY) gives each thread TX x TY cells of its tile and shrinks the CTA
//    to (16/TX) x (16/TY) threads, #CTAs unchanged.  Block coarsening
//    (bx,by, runtime) merges bx x by tiles into one CTA, threads unchanged, #CTAs / (bx*by)
//    (PAPER.md:181-185); ragged edges are masked (the paper's epilogue).
//    MODE 0 = coalescing-friendly indexing (a thread's cells are NTX apart), MODE 1 =
//    contiguous cells (TX % 4 == 0 -> 128-bit loads/stores) (Fig. 11).
//    Neighbours are read straight from global memory (L1 serves the reuse): at one step per
//    launch the kernel is HBM-bound at 12 B per cell-update.
//
//  * hs_stream<V,H>  (temporal = H >= 2), the B200 temporal-blocking family.  Each warp owns a
//    band of 32*V staged columns (V contiguous columns per lane, 128-bit accesses) and streams
//    down a chunk of rows; H time levels are kept in registers as 3-row rings and advance one
//    row per step with a lag of one row per level, so H steps of the stencil cost one HBM read
//    of T and P and one write of T'.  E/W neighbours come from warp shuffles, N/S from the
//    register rings; no shared memory and no block barriers.  The band overlaps its neighbours
//    by H columns on each side (redundant halo compute), the chunk by H rows above and below.
//    Results are bit-identical to H applications of hs_direct (same hs_cell, same operands).
#include <cuda_runtime.h>

#include <algorithm>

#include "hs_cell.cuh"
#include "rg_internal.h"

namespace rg {

__device__ __forceinline__ float4 ldg4(const float* p) {
    return __ldg(reinterpret_cast<const float4*>(p));
}
__device__ __forceinline__ void stg4(float* p, float4 v) { *reinterpret_cast<float4*>(p) = v; }

// ============================================================================ direct family
// ptxas otherwise budgets registers for 2048 resident threads (32 regs) and spills the
// coarsened variants; ask for >= 1024 resident threads (<= 64 regs) instead.
template <int TX, int TY, int MODE>
__global__ void __launch_bounds__((16 / TX) * (16 / TY),
                                  (1024 / ((16 / TX) * (16 / TY))) < 32 ? (1024 / ((16 / TX) * (16 / TY))) : 32)
    hs_direct(const float* __restrict__ tin, const float* __restrict__ pw,
              float* __restrict__ tout, int R, int C, int bx, int by, HsCoef cf, int vec_ok) {
    constexpr int NTX = 16 / TX, NTY = 16 / TY;
    const int x0 = blockIdx.x * 16 * bx;
    const int y0 = blockIdx.y * 16 * by;
    for (int b_y = 0; b_y < by; ++b_y) {
#pragma unroll
        for (int t_y = 0; t_y < TY; ++t_y) {
            const int row = y0 + b_y * 16 +
                            (MODE == 0 ? (int)threadIdx.y + t_y * NTY : (int)threadIdx.y * TY + t_y);
            if (row >= R) continue;
            const size_t rc = (size_t)row * C;
            const size_t rn = (size_t)max(row - 1, 0) * C;
            const size_t rs = (size_t)min(row + 1, R - 1) * C;
            for (int b_x = 0; b_x < bx; ++b_x) {
                const int xt = x0 + b_x * 16;
                if (MODE == 1) {
                    const int col0 = xt + (int)threadIdx.x * TX;
                    if ((TX % 4 == 0) && vec_ok && col0 + TX <= C) {
#pragma unroll
                        for (int q = 0; q < TX / 4; ++q) {
                            const int cq = col0 + 4 * q;
                            const float4 c4 = ldg4(tin + rc + cq);
                            const float4 n4 = ldg4(tin + rn + cq);
                            const float4 s4 = ldg4(tin + rs + cq);
                            const float4 p4 = ldg4(pw + rc + cq);
                            const float w = cq > 0 ? __ldg(tin + rc + cq - 1) : c4.x;
                            const float e = cq + 4 < C ? __ldg(tin + rc + cq + 4) : c4.w;
                            float4 o;
                            o.x = hs_cell(c4.x, n4.x, s4.x, c4.y, w, p4.x, cf);
                            o.y = hs_cell(c4.y, n4.y, s4.y, c4.z, c4.x, p4.y, cf);
                            o.z = hs_cell(c4.z, n4.z, s4.z, c4.w, c4.y, p4.z, cf);
                            o.w = hs_cell(c4.w, n4.w, s4.w, e, c4.z, p4.w, cf);
                            stg4(tout + rc + cq, o);
                        }
                        continue;
                    }
                }
#pragma unroll
                for (int t_x = 0; t_x < TX; ++t_x) {
                    const int col = MODE == 0 ? xt + (int)threadIdx.x + t_x * NTX
                                              : xt + (int)threadIdx.x * TX + t_x;
                    if (col >= C) continue;
                    const int cw = max(col - 1, 0), ce = min(col + 1, C - 1);
                    const float c = __ldg(tin + rc + col);
                    tout[rc + col] = hs_cell(c, __ldg(tin + rn + col), __ldg(tin + rs + col),
                                             __ldg(tin + rc + ce), __ldg(tin + rc + cw),
                                             __ldg(pw + rc + col), cf);
                }
            }
        }
    }
}

// ============================================================================ stream family
// Per-lane register state: ring[l][slot][v] holds level l (0 = input T) at three consecutive
// rows; at step s (level-0 row g0 = ystart + s) level l's newest row g0 - l sits in slot
// (s+2)%3, row g0-l-1 in (s+1)%3 and row g0-l-2 in s%3.  The step loop is unrolled by 3 so
// every ring index is a compile-time constant (no register moves).
//
// Fast path (EC = ER = false, the vast majority of warps): the band lies inside the grid with
// aligned vector access and the chunk's staged rows lie strictly inside the grid, so there are
// no bounds checks and no clamps; every branch below is warp-uniform.
//   EC: band touches a grid column edge (or vector access impossible) -> scalar, column clamp.
//   ER: chunk's staged rows reach row 0 or R-1 -> row checks and row clamp.
template <int V>
struct VecT;
template <> struct VecT<1> { typedef float T; };
template <> struct VecT<2> { typedef float2 T; };
template <> struct VecT<4> { typedef float4 T; };

template <int V, bool EC, bool ER>
__device__ __forceinline__ void hs_ld(const float* __restrict__ base, int row, int R, int C, int col0,
                                      float (&out)[V]) {
    if (ER && (row < 0 || row >= R)) {
#pragma unroll
        for (int v = 0; v < V; ++v) out[v] = 0.0f;
        return;
    }
    const float* p = base + (size_t)row * C + col0;
    if (!EC) {
        const typename VecT<V>::T t = __ldg(reinterpret_cast<const typename VecT<V>::T*>(p));
        const float* f = reinterpret_cast<const float*>(&t);
#pragma unroll
        for (int v = 0; v < V; ++v) out[v] = f[v];
    } else {
#pragma unroll
        for (int v = 0; v < V; ++v) {
            const int c = col0 + v;
            out[v] = (c >= 0 && c < C) ? __ldg(p + v) : 0.0f;
        }
    }
}

// Input rows stream through per-lane cp.async rings in shared memory (lane-private slots, so no
// barrier): the T ring holds HS_DT rows, requested HS_DT-1 steps ahead; the P ring additionally
// keeps each power row for the H steps during which levels 1..H read it (depth HsRing<H>::DP).
// Rows outside [0, R) are zero-filled (their values only feed cells that are never stored).
constexpr int HS_DT = 8;
#ifndef RG_HS_TRAP
#define RG_HS_TRAP 1  // top-halo trapezoid (hs_stream_step PRO); 0 only for A/B builds
#endif
template <int H>
struct HsRing {
    static constexpr int need = HS_DT + H;
    static constexpr int DP = need <= 8 ? 8 : (need <= 16 ? 16 : 32);
};

template <int V, bool EC>
__device__ __forceinline__ void hs_issue_row(float* dst_base, const float* __restrict__ src_base, int row, int R,
                                             int C, int col0, int sc0, int slot) {
    float* dst = dst_base + slot * 32 * V + sc0;
    const bool rok = row >= 0 && row < R;
    const float* src = src_base + (size_t)(rok ? row : 0) * C;
    if (!EC && V % 4 == 0) {
#pragma unroll
        for (int q = 0; q < V / 4; ++q)
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"((uint32_t)__cvta_generic_to_shared(dst + 4 * q)),
                         "l"(src + col0 + 4 * q), "r"(rok ? 16 : 0));
    } else if (!EC && V == 2) {
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"((uint32_t)__cvta_generic_to_shared(dst)),
                     "l"(src + col0), "r"(rok ? 8 : 0));
    } else {
#pragma unroll
        for (int v = 0; v < V; ++v) {
            const int c = col0 + v;
            const bool ok = rok && c >= 0 && c < C;
            asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;\n" ::"r"((uint32_t)__cvta_generic_to_shared(dst + v)),
                         "l"(ok ? src + c : src_base), "r"(ok ? 4 : 0));
        }
    }
}

template <int V>
__device__ __forceinline__ void hs_read_row(const float* base, int sc0, int slot, float (&o)[V]) {
    const float* p = base + slot * 32 * V + sc0;
    if (V % 4 == 0) {
#pragma unroll
        for (int q = 0; q < V / 4; ++q) {
            const float4 t = reinterpret_cast<const float4*>(p)[q];
            o[(4 * q) % V] = t.x; o[(4 * q + 1) % V] = t.y; o[(4 * q + 2) % V] = t.z; o[(4 * q + 3) % V] = t.w;
        }
    } else {
#pragma unroll
        for (int v = 0; v < V; ++v) o[v] = p[v];
    }
}

// Request the rows step `s` will consume: T row ystart+s into slot s % HS_DT, P row ystart+s-1
// into slot s % DP (one commit group per step).  Fast path (interior band and chunk, every
// requested row inside the grid): running per-lane source pointers advanced by one row per
// request and lane-constant shared-memory bases, so a request costs two 128-bit copies and a
// few integer operations instead of clamped row arithmetic.
template <int V, int H, bool EC, bool ER>
__device__ __forceinline__ void hs_issue_step(float* tring, float* pring, const float* __restrict__ tin,
                                              const float* __restrict__ pw, int s, int ystart, int R, int C,
                                              int col0, int sc0, const float*& tsrc, const float*& psrc) {
    if (!EC && !ER && V % 4 == 0) {
        constexpr int DP = HsRing<H>::DP;
        const uint32_t td = (uint32_t)__cvta_generic_to_shared(tring + sc0) + (uint32_t)((s & (HS_DT - 1)) * 32 * V * 4);
        const uint32_t pd = (uint32_t)__cvta_generic_to_shared(pring + sc0) + (uint32_t)((s & (DP - 1)) * 32 * V * 4);
#pragma unroll
        for (int q = 0; q < V / 4; ++q) {
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(td + 16 * q), "l"(tsrc + 4 * q));
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(pd + 16 * q), "l"(psrc + 4 * q));
        }
        tsrc += C;
        psrc += C;
    } else {
        hs_issue_row<V, EC>(tring, tin, ystart + s, R, C, col0, sc0, s & (HS_DT - 1));
        hs_issue_row<V, EC>(pring, pw, ystart + s - 1, R, C, col0, sc0, s & (HsRing<H>::DP - 1));
    }
    asm volatile("cp.async.commit_group;\n" ::);
}

// PRO (the first 2H steps of a chunk): level l+1 is skipped at steps s < 2l+2.  Level L's rows
// above y0-H+L are never needed (the output rows [y0, y1) depend on level L only through rows
// [y0-H+L, y1+H-L)), and a skipped row is only ever read by rows that are skipped too, so the
// stored results are unchanged; this trims the chunk's top halo from a rectangle of 2H rows per
// level to the trapezoid (H(H+1) fewer row updates per chunk).  The bottom halo is already
// trapezoidal through the one-row lag per level.
template <int V, int H, int K, bool EC, bool ER, bool PRO>
__device__ __forceinline__ void hs_stream_step(float (&ring)[H][3][V], float* tring, float* pring,
                                               const float* __restrict__ tin, const float* __restrict__ pw,
                                               float* __restrict__ tout, int s, int ystart, int R, int C, int ylo,
                                               int yhi, int sc0, int col0, const HsCoef& cf,
                                               const float*& tsrc, const float*& psrc, float*& optr) {
    constexpr int S0 = K % 3, S1 = (K + 1) % 3, S2 = (K + 2) % 3;
    constexpr int DP = HsRing<H>::DP;
    const int g0 = ystart + s;
    // this step's rows have landed once at most HS_DT-2 later groups are pending
    asm volatile("cp.async.wait_group %0;\n" ::"n"(HS_DT - 2));
    hs_read_row<V>(tring, sc0, s & (HS_DT - 1), ring[0][S2]);  // level 0 = T row g0
    hs_issue_step<V, H, EC, ER>(tring, pring, tin, pw, s + HS_DT - 1, ystart, R, C, col0, sc0, tsrc, psrc);

#pragma unroll
    for (int l = 0; l < H; ++l) {
        if (PRO && s < 2 * l + 2) break;  // levels l+1.. are all above their trapezoid (warp-uniform)
        const int g = g0 - l - 1;  // row computed by level l+1 (its power row was level 1's at step s-l)
        float pv[V];
        hs_read_row<V>(pring, sc0, (s - l) & (DP - 1), pv);
        const bool top = ER && (g == 0), bot = ER && (g == R - 1);
        const float wnb = __shfl_up_sync(0xffffffffu, ring[l][S1][V - 1], 1);
        const float enb = __shfl_down_sync(0xffffffffu, ring[l][S1][0], 1);
        float res[V];
        float ew[V];
#pragma unroll
        for (int v = 0; v < V; ++v) {
            const float c = ring[l][S1][v];
            float w = v > 0 ? ring[l][S1][v > 0 ? v - 1 : 0] : wnb;
            float e = v < V - 1 ? ring[l][S1][v < V - 1 ? v + 1 : 0] : enb;
            if (EC) {
                const int col = col0 + v;
                if (col == 0) w = c;
                if (col == C - 1) e = c;
            }
            ew[v] = __fadd_rn(e, w);
        }
        if constexpr (V % 2 == 0) {
            // column pairs through the packed FP32x2 pipe (FADD2/FFMA2): same per-element
            // operations and roundings as hs_cell, half the issue slots (hs_cell2)
#pragma unroll
            for (int q = 0; q < V / 2; ++q) {
                const int v0 = 2 * q, v1 = 2 * q + 1;
                const float2 c2 = make_float2(ring[l][S1][v0], ring[l][S1][v1]);
                const float2 n2 = top ? c2 : make_float2(ring[l][S0][v0], ring[l][S0][v1]);
                const float2 s2 = bot ? c2 : make_float2(ring[l][S2][v0], ring[l][S2][v1]);
                const float2 r = hs_cell2(c2, n2, s2, make_float2(ew[v0], ew[v1]), make_float2(pv[v0], pv[v1]), cf);
                res[v0] = r.x;
                res[v1] = r.y;
            }
        } else {
#pragma unroll
            for (int v = 0; v < V; ++v) {
                const float c = ring[l][S1][v];
                const float n = top ? c : ring[l][S0][v];
                const float s_ = bot ? c : ring[l][S2][v];
                res[v] = hs_cell_ew(c, n, s_, ew[v], pv[v], cf);
            }
        }
        if (l + 1 < H) {
#pragma unroll
            for (int v = 0; v < V; ++v) ring[l + 1 < H ? l + 1 : 0][S2][v] = res[v];
        } else if ((!PRO && RG_HS_TRAP) || (g >= ylo && g < yhi)) {
            // (the steady loop runs steps 2H <= s <= nsteps - 1 only, whose level-H rows
            // y0 - 2H + s all lie in [y0, y1): no row test there)
            // level H: write the lane's cells that lie in the band's output columns
            constexpr int s_lo = H, s_hi = 32 * V - H;  // staged-column range of the output
            float* orow = optr;  // = tout + g * C + col0 (running pointer: no per-step 64-bit multiply)
            if constexpr (!EC && (H % V == 0) && V <= 4) {
                if (sc0 >= s_lo && sc0 < s_hi) {
                    typename VecT<V>::T t;
                    float* f = reinterpret_cast<float*>(&t);
#pragma unroll
                    for (int v = 0; v < V; ++v) f[v] = res[v];
                    *reinterpret_cast<typename VecT<V>::T*>(orow) = t;
                }
            } else if constexpr (!EC && V % 4 == 0 && H % 4 == 0) {
                // 128-bit pieces: each lies wholly inside or outside the output range
#pragma unroll
                for (int q = 0; q < V / 4; ++q)
                    if (sc0 + 4 * q >= s_lo && sc0 + 4 * q < s_hi)
                        *reinterpret_cast<float4*>(orow + 4 * q) =
                            make_float4(res[4 * q], res[4 * q + 1], res[4 * q + 2], res[4 * q + 3]);
            } else {
#pragma unroll
                for (int v = 0; v < V; ++v) {
                    const int col = col0 + v;
                    if (sc0 + v >= s_lo && sc0 + v < s_hi && col >= 0 && col < C) orow[v] = res[v];
                }
            }
        }
    }
    optr += C;
}

template <int V, int H, bool EC, bool ER>
__device__ __forceinline__ void hs_stream_body(const float* __restrict__ tin,
                                               const float* __restrict__ pw,
                                               float* __restrict__ tout, float* tring, float* pring, int R,
                                               int C, int y0, int y1, int sc0, int col0, const HsCoef& cf) {
    float ring[H][3][V];
#pragma unroll
    for (int l = 0; l < H; ++l)
#pragma unroll
        for (int k = 0; k < 3; ++k)
#pragma unroll
            for (int v = 0; v < V; ++v) ring[l][k][v] = 0.0f;
    const int ystart = y0 - H;
    const int nsteps = (y1 - y0) + 2 * H;
    // fast-path source pointers (only dereferenced when !EC && !ER: all requested rows exist)
    const float* tsrc = tin + (size_t)max(ystart, 0) * C + col0;
    const float* psrc = pw + (size_t)max(ystart - 1, 0) * C + col0;
    // output row of level H at step s: ystart + s - H (only dereferenced inside [y0, y1))
    float* optr = tout + (ptrdiff_t)(ystart - H) * C + col0;
#pragma unroll
    for (int k = 0; k < HS_DT - 1; ++k)
        hs_issue_step<V, H, EC, ER>(tring, pring, tin, pw, k, ystart, R, C, col0, sc0, tsrc, psrc);
    int s = 0;
    // prologue: the top-halo trapezoid (levels switched on two steps apart)
    for (; RG_HS_TRAP && s + 3 <= nsteps && s < 2 * H; s += 3) {
        hs_stream_step<V, H, 0, EC, ER, true>(ring, tring, pring, tin, pw, tout, s, ystart, R, C, y0, y1, sc0, col0, cf, tsrc, psrc, optr);
        hs_stream_step<V, H, 1, EC, ER, true>(ring, tring, pring, tin, pw, tout, s + 1, ystart, R, C, y0, y1, sc0, col0, cf, tsrc, psrc, optr);
        hs_stream_step<V, H, 2, EC, ER, true>(ring, tring, pring, tin, pw, tout, s + 2, ystart, R, C, y0, y1, sc0, col0, cf, tsrc, psrc, optr);
    }
    for (; s + 3 <= nsteps; s += 3) {
        hs_stream_step<V, H, 0, EC, ER, false>(ring, tring, pring, tin, pw, tout, s, ystart, R, C, y0, y1, sc0, col0, cf, tsrc, psrc, optr);
        hs_stream_step<V, H, 1, EC, ER, false>(ring, tring, pring, tin, pw, tout, s + 1, ystart, R, C, y0, y1, sc0, col0, cf, tsrc, psrc, optr);
        hs_stream_step<V, H, 2, EC, ER, false>(ring, tring, pring, tin, pw, tout, s + 2, ystart, R, C, y0, y1, sc0, col0, cf, tsrc, psrc, optr);
    }
    if (s < nsteps) hs_stream_step<V, H, 0, EC, ER, true>(ring, tring, pring, tin, pw, tout, s, ystart, R, C, y0, y1, sc0, col0, cf, tsrc, psrc, optr);
    if (s + 1 < nsteps) hs_stream_step<V, H, 1, EC, ER, true>(ring, tring, pring, tin, pw, tout, s + 1, ystart, R, C, y0, y1, sc0, col0, cf, tsrc, psrc, optr);
    asm volatile("cp.async.wait_group 0;\n" ::);  // drain before the rings are reused
}

// One warp per CTA: every branch condition derives from blockIdx and kernel arguments only, so
// the compiler sees it as warp-uniform and the shuffles need no convergence handling.  Block
// coarsening along x (bands_per_cta) makes the warp process several adjacent bands in turn;
// block coarsening along y is the chunk height (rows streamed per CTA).
template <int V, int H, int OCC>
__global__ void __launch_bounds__(32, OCC)
    hs_stream(const float* __restrict__ tin, const float* __restrict__ pw,
              float* __restrict__ tout, int R, int C, int chunk, int bands_per_cta, HsCoef cf,
              int vec_ok) {
    constexpr int SW = 32 * V;
    constexpr int OW = SW - 2 * H;
    static_assert(OW > 0, "band narrower than its halo");
    asm volatile("griddepcontrol.wait;" ::: "memory");  // launched as a programmatic dependent
    const int sc0 = (int)threadIdx.x * V;
    const int y0 = blockIdx.y * chunk;
    const int y1 = min(y0 + chunk, R);
    // rows computed: [y0-H, y1+H); ER selects the row-clamp path near the grid's top/bottom
    // (rows requested: [y0-H-1, y1+H+HS_DT-1), the prefetch running HS_DT-1 rows past the last step)
    const bool er = (y0 - H - 1 < 0) || (y1 + H + HS_DT - 1 > R);
    __shared__ __align__(16) float tring[HS_DT * 32 * V];
    __shared__ __align__(16) float pring[HsRing<H>::DP * 32 * V];
    for (int bi = 0; bi < bands_per_cta; ++bi) {
        const int band = blockIdx.x * bands_per_cta + bi;
        if (band * OW >= C) return;
        const int bstart = band * OW - H;
        const int col0 = bstart + sc0;
        const bool ec = !vec_ok || bstart < 0 || bstart + SW > C;
        if (!ec && !er)
            hs_stream_body<V, H, false, false>(tin, pw, tout, tring, pring, R, C, y0, y1, sc0, col0, cf);
        else if (ec && !er)
            hs_stream_body<V, H, true, false>(tin, pw, tout, tring, pring, R, C, y0, y1, sc0, col0, cf);
        else if (!ec && er)
            hs_stream_body<V, H, false, true>(tin, pw, tout, tring, pring, R, C, y0, y1, sc0, col0, cf);
        else
            hs_stream_body<V, H, true, true>(tin, pw, tout, tring, pring, R, C, y0, y1, sc0, col0, cf);
    }
}

// ============================================================================ registry
namespace hotspot {

typedef void (*DirectFn)(const float*, const float*, float*, int, int, int, int, HsCoef, int);
typedef void (*StreamFn)(const float*, const float*, float*, int, int, int, int, HsCoef, int);

struct DirectVariant { int tx, ty, mode; DirectFn fn; const char* key; };
struct StreamVariant { int v, h, occ; StreamFn fn; const char* key; };

#define RG_HSD(TX, TY, M) {TX, TY, M, hs_direct<TX, TY, M>, "void rg::hs_direct<" #TX ", " #TY ", " #M ">"}
#define RG_HSD2(TX, TY) RG_HSD(TX, TY, 0), RG_HSD(TX, TY, 1)
static const DirectVariant kDirect[] = {
    RG_HSD2(1, 1),  RG_HSD2(1, 2), RG_HSD2(1, 4), RG_HSD2(1, 8), RG_HSD2(1, 16),
    RG_HSD2(2, 1),  RG_HSD2(2, 2), RG_HSD2(2, 4), RG_HSD2(2, 8), RG_HSD2(2, 16),
    RG_HSD2(4, 1),  RG_HSD2(4, 2), RG_HSD2(4, 4), RG_HSD2(4, 8),
    RG_HSD2(8, 1),  RG_HSD2(8, 2), RG_HSD2(8, 4),
    RG_HSD2(16, 1), RG_HSD2(16, 2),
};
#undef RG_HSD2
#undef RG_HSD

#define RG_HSS(V, H, O) {V, H, O, hs_stream<V, H, O>, "void rg::hs_stream<" #V ", " #H ", " #O ">"}
static const StreamVariant kStream[] = {
    RG_HSS(4, 2, 16), RG_HSS(4, 2, 24),
    RG_HSS(4, 4, 12), RG_HSS(4, 4, 16), RG_HSS(4, 4, 20), RG_HSS(4, 4, 24),
    RG_HSS(4, 6, 10), RG_HSS(4, 6, 12), RG_HSS(4, 6, 16),
    RG_HSS(4, 8, 8), RG_HSS(4, 8, 10), RG_HSS(4, 8, 12), RG_HSS(4, 8, 14), RG_HSS(4, 8, 16),
    RG_HSS(2, 4, 16), RG_HSS(2, 4, 24), RG_HSS(2, 4, 32),
    RG_HSS(2, 8, 12), RG_HSS(2, 8, 16), RG_HSS(2, 8, 20), RG_HSS(2, 8, 24),
    RG_HSS(2, 12, 12), RG_HSS(2, 12, 16),
    RG_HSS(2, 16, 8), RG_HSS(2, 16, 12),
    RG_HSS(1, 4, 16), RG_HSS(1, 8, 16),
};
#undef RG_HSS

const DirectVariant* find_direct(int tx, int ty, int mode) {
    for (const auto& v : kDirect)
        if (v.tx == tx && v.ty == ty && v.mode == mode) return &v;
    return nullptr;
}
// occ == 0 selects the first instantiation of (V, H) in kStream (ordered by preference).
const StreamVariant* find_stream(int v_, int h, int occ) {
    for (const auto& v : kStream)
        if (v.v == v_ && v.h == h && (occ == 0 || v.occ == occ)) return &v;
    return nullptr;
}

static bool is_div16(int t) { return t == 1 || t == 2 || t == 4 || t == 8 || t == 16; }

// Host-only legality check (no CUDA call).  Fills the variant pointers.
rodinia_status check(const rodinia_granularity& g, int64_t R, int64_t C,
                     const DirectVariant** dv, const StreamVariant** sv) {
    *dv = nullptr; *sv = nullptr;
    if (g.thread_x < 1 || g.thread_y < 1 || g.block_x < 1 || g.block_y < 1 || g.temporal < 1)
        return set_error(RODINIA_E_ILLEGAL_FACTOR, "hotspot: factors must be >= 1 (%s)", gran_str(g).c_str());
    if (g.index_mode != 0 && g.index_mode != 1)
        return set_error(RODINIA_E_ILLEGAL_FACTOR, "hotspot: index_mode must be 0 or 1");
    const bool stream = (g.flags & RODINIA_STREAM) != 0;
    if (!stream) {
        if (g.temporal != 1)
            return set_error(RODINIA_E_ILLEGAL_FACTOR,
                             "hotspot: the direct family fuses one step per launch (temporal=1); "
                             "set RODINIA_STREAM for temporal blocking");
        if (!is_div16(g.thread_x) || !is_div16(g.thread_y))
            return set_error(RODINIA_E_ILLEGAL_FACTOR,
                             "hotspot: thread factors must divide the 16x16 tile (PAPER.md:237)");
        if (g.block_x > 4096 || g.block_y > 4096)
            return set_error(RODINIA_E_ILLEGAL_FACTOR, "hotspot: block factor too large");
        const int64_t gy = ((R + 15) / 16 + g.block_y - 1) / g.block_y;
        if (gy > 65535)
            return set_error(RODINIA_E_ILLEGAL_FACTOR, "hotspot: grid.y %lld > 65535; raise block_y", (long long)gy);
        *dv = find_direct(g.thread_x, g.thread_y, g.index_mode);
        if (!*dv)
            return set_error(RODINIA_E_NOT_BUILT, "hotspot: direct variant %s not instantiated", gran_str(g).c_str());
    } else {
        if (g.flags & RODINIA_FAITHFUL)
            return set_error(RODINIA_E_ILLEGAL_FACTOR, "hotspot: the stream family is not a faithful-mode variant");
        if (g.thread_y != 1 || g.index_mode != 1)
            return set_error(RODINIA_E_NOT_BUILT, "hotspot: stream family needs thread_y=1, index_mode=1");
        if (g.temporal < 2)
            return set_error(RODINIA_E_ILLEGAL_FACTOR, "hotspot: stream family needs temporal >= 2");
        if (g.block_x > 4096)
            return set_error(RODINIA_E_ILLEGAL_FACTOR, "hotspot: stream block_x too large");
        const int64_t chunk = 16 * (int64_t)g.block_y;
        if ((R + chunk - 1) / chunk > 65535)
            return set_error(RODINIA_E_ILLEGAL_FACTOR, "hotspot: too many row chunks; raise block_y");
        *sv = find_stream(g.thread_x, g.temporal, RODINIA_OCC_OF(g.flags));
        if (!*sv)
            return set_error(RODINIA_E_NOT_BUILT, "hotspot: stream variant %s not instantiated", gran_str(g).c_str());
    }
    // compile-time filter at the boundary
    return *dv ? boundary_filter(RODINIA_HOTSPOT, (*dv)->key, (16 / (*dv)->tx) * (16 / (*dv)->ty), 0, g.flags)
               : boundary_filter(RODINIA_HOTSPOT, (*sv)->key, 32, 0, g.flags);
}

static void launch_direct(const DirectVariant* dv, int bx, int by, const float* tin, const float* p,
                          float* tout, int R, int C, const HsCoef& cf, cudaStream_t s) {
    const int tiles_x = (C + 15) / 16, tiles_y = (R + 15) / 16;
    dim3 grid((tiles_x + bx - 1) / bx, (tiles_y + by - 1) / by);
    dim3 block(16 / dv->tx, 16 / dv->ty);
    const int vec_ok = (C % 4 == 0) &&
                       ((reinterpret_cast<uintptr_t>(tin) | reinterpret_cast<uintptr_t>(p) |
                         reinterpret_cast<uintptr_t>(tout)) % 16 == 0);
    dv->fn<<<grid, block, 0, s>>>(tin, p, tout, R, C, bx, by, cf, vec_ok);
    count_launch();
}

static void launch_stream(const StreamVariant* sv, int bx, int by, const float* tin, const float* p,
                          float* tout, int R, int C, const HsCoef& cf, cudaStream_t s) {
    const int ow = 32 * sv->v - 2 * sv->h;
    const int bands = (C + ow - 1) / ow;
    const int chunk = 16 * by;
    dim3 grid((bands + bx - 1) / bx, (R + chunk - 1) / chunk);
    // vector access needs every lane's first column aligned to V floats
    const int vec_ok = (C % sv->v == 0) && (sv->h % sv->v == 0) &&
                       ((reinterpret_cast<uintptr_t>(tin) | reinterpret_cast<uintptr_t>(p) |
                         reinterpret_cast<uintptr_t>(tout)) % (4 * sv->v) == 0);
    // programmatic dependent of the preceding kernel (hs_stream waits with griddepcontrol.wait
    // before touching memory): the launch of step-block k+1 overlaps the drain of step-block k
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = dim3(32);
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaLaunchKernelEx(&cfg, sv->fn, tin, p, tout, R, C, chunk, bx, cf, vec_ok);
    count_launch();
}

// ---------------------------------------------------------------- state conversions
// y = x - a (T -> u), y = x * a (P -> kP), y = x + a (u -> T); elementwise, grid-stride,
// 128-bit when all pointers are 16-byte aligned.  In place is allowed (x == y).
template <int OP>
__device__ __forceinline__ float hs_conv1(float x, float a) {
    return OP == 0 ? __fsub_rn(x, a) : (OP == 1 ? __fmul_rn(x, a) : __fadd_rn(x, a));
}
template <int OP>
__global__ void __launch_bounds__(256) hs_convert(const float* x, float* y, int64_t n, float a, int vec) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (vec) {
        const int64_t n4 = n / 4;
        for (int64_t j = i; j < n4; j += stride) {
            float4 v = reinterpret_cast<const float4*>(x)[j];
            v.x = hs_conv1<OP>(v.x, a); v.y = hs_conv1<OP>(v.y, a);
            v.z = hs_conv1<OP>(v.z, a); v.w = hs_conv1<OP>(v.w, a);
            reinterpret_cast<float4*>(y)[j] = v;
        }
        i += n4 * 4;
    }
    for (; i < n; i += stride) y[i] = hs_conv1<OP>(x[i], a);
}

void convert(const float* x, float* y, int64_t n, int op, float a, cudaStream_t s) {
    if (n <= 0) return;
    const int vec = ((reinterpret_cast<uintptr_t>(x) | reinterpret_cast<uintptr_t>(y)) % 16) == 0;
    const int64_t want = (n / 4 + 255) / 256 + 1;
    const int grid = (int)std::min<int64_t>(want, 148 * 8);
    if (op == 0) hs_convert<0><<<grid, 256, 0, s>>>(x, y, n, a, vec);
    else if (op == 1) hs_convert<1><<<grid, 256, 0, s>>>(x, y, n, a, vec);
    else hs_convert<2><<<grid, 256, 0, s>>>(x, y, n, a, vec);
    count_launch();
}

int num_launches(int iters, const StreamVariant* sv) {
    const int h = sv ? sv->h : 1;
    return iters / h + iters % h;  // remainder steps run one per launch (direct family)
}

// Run `iters` steps in state space on a (R x C) buffer from `usrc` into `udst`, ping-ponging
// through `uscr` (`usrc` may be `uscr` when num_launches() is odd, or `udst` when it is even).
// The granularity has been validated by check().  Neighbour rows are clamped to the buffer,
// so the same routine serves whole grids and halo'd slabs.
rodinia_status run(const float* usrc, const float* kp, float* udst, float* uscr, int R, int C,
                   int iters, const HsCoef& cf, const rodinia_granularity& g,
                   const DirectVariant* dv, const StreamVariant* sv, cudaStream_t s) {
    if (iters == 0) {
        if (udst != usrc)
            RG_CUDA(cudaMemcpyAsync(udst, usrc, (size_t)R * C * sizeof(float), cudaMemcpyDeviceToDevice, s));
        return RODINIA_OK;
    }
    const int h = sv ? sv->h : 1;
    const int nfull = iters / h;
    const int launches = num_launches(iters, sv);
    const DirectVariant* remv = find_direct(4, 1, 1);
    int left = launches;
    const float* src = usrc;
    int done = 0;
    while (left > 0) {
        float* dst = ((left - 1) % 2 == 0) ? udst : uscr;
        if (sv && done < nfull) {
            ktime_begin(s);
            launch_stream(sv, g.block_x, g.block_y, src, kp, dst, R, C, cf, s);
            ktime_end(s);
            ++done;
        } else if (dv) {
            ktime_begin(s);
            launch_direct(dv, g.block_x, g.block_y, src, kp, dst, R, C, cf, s);
            ktime_end(s);
        } else {
            launch_direct(remv, 1, 1, src, kp, dst, R, C, cf, s);
        }
        src = dst;
        --left;
    }
    RG_CUDA(cudaGetLastError());
    return RODINIA_OK;
}

// Whole solve from temperatures: T -> u (into the buffer the first launch does not write),
// P -> kP (into `kp`), `iters` steps, u -> T in place in `tout`.  `scr` and `kp` are R x C
// scratch buffers distinct from every operand.
rodinia_status solve(const float* tin, const float* p, float* tout, float* scr, float* kp, int R, int C,
                     int iters, const rodinia_hotspot_coeffs& cc, const rodinia_granularity& g,
                     const DirectVariant* dv, const StreamVariant* sv, cudaStream_t s) {
    const int64_t n = (int64_t)R * C;
    if (iters == 0) {
        RG_CUDA(cudaMemcpyAsync(tout, tin, (size_t)n * sizeof(float), cudaMemcpyDeviceToDevice, s));
        return RODINIA_OK;
    }
    const HsCoef cf = hs_derive(cc.k, cc.rx, cc.ry, cc.rz);
    float* u0 = (num_launches(iters, sv) % 2 == 1) ? scr : tout;
    convert(tin, u0, n, 0, cc.amb, s);
    convert(p, kp, n, 1, cc.k, s);
    RG_TRY(run(u0, kp, tout, scr, R, C, iters, cf, g, dv, sv, s));
    convert(tout, tout, n, 2, cc.amb, s);
    RG_CUDA(cudaGetLastError());
    return RODINIA_OK;
}

int num_variants() { return (int)(sizeof(kDirect) / sizeof(kDirect[0]) + sizeof(kStream) / sizeof(kStream[0])); }

int temporal_of(const StreamVariant* sv) { return sv ? sv->h : 1; }

// Describe variant i: granularity (block factors 1), kernel pointer, key, threads per CTA.
void variant_info(int i, rodinia_granularity* g, const void** fn, const char** key, int* threads) {
    const int nd = (int)(sizeof(kDirect) / sizeof(kDirect[0]));
    if (i < nd) {
        const auto& v = kDirect[i];
        *g = gran(v.tx, v.ty, 1, 1, 1, v.mode);
        *fn = (const void*)v.fn;
        *key = v.key;
        *threads = (16 / v.tx) * (16 / v.ty);
    } else {
        const auto& v = kStream[i - nd];
        *g = gran(v.v, 1, 1, 4, v.h, 1, RODINIA_STREAM | RODINIA_OCC(v.occ));
        *fn = (const void*)v.fn;
        *key = v.key;
        *threads = 32;
    }
}

}  // namespace hotspot
}  // namespace rg

// pathfinder.cu -- granularity-parameterised pathfinder (min-cost path DP) for sm_100a.
//
// Operation: Rodinia pathfinder `dynproc_kernel` (DESIGN.md §3 P1-P6):
//   prev = wall[0]; next[j] = wall[r][j] + min(prev[j-1], prev[j], prev[j+1]) over existing
//   indices, r = 1..R-1; result = prev.  int32, bit-exact.
//
// Kernel pf_pyramid<CELLS,MODE>: the Rodinia pyramid (h DP rows per launch, a band of
// columns per CTA that overlaps its neighbours by h columns per side), re-sized for B200.
//  * thread coarsening t and block coarsening b: the original CTA is 256 threads x 1 column.
//    A thread owns CELLS = t*b columns; the CTA has ceil(256/t) threads rounded up to a warp
//    (t = 1..8 need not divide 256 outside FAITHFUL mode, reading P5) and covers about
//    256*b columns.  MODE 0 strides a thread's columns by the thread count (coalescing-
//    friendly), MODE 1 makes them contiguous.
//  * Neighbour exchange per DP row: in-thread neighbours from registers, cross-thread ones
//    from warp shuffles (MODE 1) and a per-warp edge array in shared memory (one barrier per
//    row, double-buffered by row parity).  Edge columns of the grid use the cell's own value
//    (min(x, x) = x), which is the "existing indices only" rule without sentinels.
//  * Launches are chained with programmatic dependent launch (PDL): the next launch starts
//    its prologue (wall prefetch) while the previous one drains.
#include <cuda_runtime.h>
#include <limits.h>
#include <string.h>

#include <algorithm>

#include <vector>

#include "rg_internal.h"

namespace rg {

template <int CELLS, int MODE>
__global__ void __launch_bounds__(256)
    pf_pyramid(const int32_t* __restrict__ wall, const int32_t* __restrict__ prev_in,
               int32_t* __restrict__ next_out, int R, int C, int r0, int h, int band_out, int vec_ok) {
    (void)vec_ok;  // scalar accesses only
    // staged band: columns [b0 - h, b0 - h + NT*CELLS), outputs [b0, b0 + band_out)
    extern __shared__ int32_t pf_edges[];  // [2][nwarps][2]
    const int nt = blockDim.x;
    const int nwarps = nt >> 5;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int b0 = blockIdx.x * band_out;
    const int s0 = b0 - h;
    int col[CELLS];
#pragma unroll
    for (int k = 0; k < CELLS; ++k) col[k] = MODE == 1 ? s0 + tid * CELLS + k : s0 + tid + k * nt;

    // prologue independent of the previous launch: first wall row of this launch
    int32_t wnext[CELLS];
    const int32_t* wrow = wall + (size_t)(r0 + 1) * C;
#pragma unroll
    for (int k = 0; k < CELLS; ++k) wnext[k] = (col[k] >= 0 && col[k] < C) ? __ldg(wrow + col[k]) : 0;
#if __CUDA_ARCH__ >= 900
    cudaGridDependencySynchronize();  // PDL: prev_in is produced by the previous launch
#endif
    int32_t v[CELLS];
#pragma unroll
    for (int k = 0; k < CELLS; ++k) v[k] = (col[k] >= 0 && col[k] < C) ? prev_in[col[k]] : 0;

    for (int i = 0; i < h; ++i) {
        const int r = r0 + 1 + i;
        int32_t w[CELLS];
#pragma unroll
        for (int k = 0; k < CELLS; ++k) w[k] = wnext[k];
        if (i + 1 < h) {
            const int32_t* wr = wall + (size_t)(r + 1) * C;
#pragma unroll
            for (int k = 0; k < CELLS; ++k) wnext[k] = (col[k] >= 0 && col[k] < C) ? __ldg(wr + col[k]) : 0;
        }
        int32_t left[CELLS], right[CELLS];
        if (MODE == 1) {
            // contiguous: in-thread neighbours; thread edges via shuffles / smem
            int32_t lnb = __shfl_up_sync(0xffffffffu, v[CELLS - 1], 1);
            int32_t rnb = __shfl_down_sync(0xffffffffu, v[0], 1);
            if (nwarps > 1) {
                int32_t* e = pf_edges + (i & 1) * nwarps * 2;
                if (lane == 0) e[warp * 2 + 0] = v[0];
                if (lane == 31) e[warp * 2 + 1] = v[CELLS - 1];
                __syncthreads();
                if (lane == 0 && warp > 0) lnb = e[(warp - 1) * 2 + 1];
                if (lane == 31 && warp + 1 < nwarps) rnb = e[(warp + 1) * 2 + 0];
            }
#pragma unroll
            for (int k = 0; k < CELLS; ++k) {
                left[k] = k > 0 ? v[k > 0 ? k - 1 : 0] : lnb;
                right[k] = k < CELLS - 1 ? v[k < CELLS - 1 ? k + 1 : 0] : rnb;
            }
        } else {
            // strided: a thread's columns are nt apart; the neighbours of column c live in
            // threads tid-1 / tid+1 (same k), wrapping to the previous / next k at the ends.
            int32_t up[CELLS], dn[CELLS];
#pragma unroll
            for (int k = 0; k < CELLS; ++k) {
                up[k] = __shfl_up_sync(0xffffffffu, v[k], 1);
                dn[k] = __shfl_down_sync(0xffffffffu, v[k], 1);
            }
            int32_t* e = pf_edges + (i & 1) * nwarps * 2 * CELLS;
            if (lane == 0)
#pragma unroll
                for (int k = 0; k < CELLS; ++k) e[(warp * 2 + 0) * CELLS + k] = v[k];
            if (lane == 31)
#pragma unroll
                for (int k = 0; k < CELLS; ++k) e[(warp * 2 + 1) * CELLS + k] = v[k];
            __syncthreads();
#pragma unroll
            for (int k = 0; k < CELLS; ++k) {
                int32_t l = up[k], rr = dn[k];
                if (lane == 0)
                    l = warp > 0 ? e[((warp - 1) * 2 + 1) * CELLS + k]
                                 : (k > 0 ? e[((nwarps - 1) * 2 + 1) * CELLS + (k > 0 ? k - 1 : 0)] : 0);
                if (lane == 31)
                    rr = warp + 1 < nwarps ? e[((warp + 1) * 2 + 0) * CELLS + k]
                                           : (k + 1 < CELLS ? e[0 * CELLS + (k + 1 < CELLS ? k + 1 : 0)] : 0);
                left[k] = l;
                right[k] = rr;
            }
        }
#pragma unroll
        for (int k = 0; k < CELLS; ++k) {
            const int c = col[k];
            const int32_t l = c > 0 ? left[k] : v[k];
            const int32_t rr = c < C - 1 ? right[k] : v[k];
            const int32_t m = min(min(l, v[k]), rr);
            v[k] = (c >= 0 && c < C) ? w[k] + m : 0;
        }
    }
#pragma unroll
    for (int k = 0; k < CELLS; ++k) {
        const int c = col[k];
        if (c >= b0 && c < b0 + band_out && c < C) next_out[c] = v[k];
    }
    // only writes issued before the trigger are visible to the dependent launch
#if __CUDA_ARCH__ >= 900
    cudaTriggerProgrammaticLaunchCompletion();
#endif
}

// ------------------------------------------------------------------ warp-band family
// pf_band<CELLS> (flags RODINIA_STREAM): one warp per CTA owns a band of 32*CELLS contiguous
// columns (CELLS contiguous ints per lane, 128-bit accesses) and runs all h rows of a launch
// without any block barrier: row neighbours come from registers and two warp shuffles.  Wall
// rows stream through a per-lane cp.async ring in shared memory PfRing::D-1 rows ahead.  The band's
// halo is h rounded up to 4 columns per side (keeps 16-byte alignment).
// ring depth (rows in flight); deeper rings (16-32) were measured slower (longer prologue)
#ifndef RG_PF_D
#define RG_PF_D 8  // A/B builds only (tools/build_lib.py --define RG_PF_D=16)
#endif
template <int CELLS>
struct PfRing { static constexpr int D = RG_PF_D * CELLS <= 256 ? RG_PF_D : 256 / CELLS; };  // <= 32 KiB static smem

// shared-memory offset (ints) of cell k of `lane` in ring slot `slot`: [slot][q][lane][4] for
// CELLS % 4 == 0, [slot][lane][2] for 2-cell lanes (64-bit accesses, also conflict free)
template <int CELLS>
__device__ __forceinline__ int pf_off(int slot, int lane, int k) {
    if constexpr (CELLS % 4 == 0) return (slot * (CELLS / 4) * 32 + lane) * 4 + (k / 4) * 128 + (k % 4);
    else return (slot * 32 + lane) * CELLS + k;
}

template <int CELLS, bool EC>
__device__ __forceinline__ void pf_issue(int32_t* ring, const int32_t* __restrict__ wall, int row, int C,
                                         int col0, int lane, int slot) {
    // layout [slot][q][lane][4]: for a fixed 16-byte chunk q the 32 lanes are contiguous, so the
    // 128-bit shared stores and loads are bank-conflict free for any CELLS
    int32_t* dst = ring + pf_off<CELLS>(slot, lane, 0);
    const int32_t* src = wall + (size_t)row * C;
    if (!EC && CELLS == 2) {
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"((uint32_t)__cvta_generic_to_shared(dst)),
                     "l"(src + col0));
    } else if (!EC) {
#pragma unroll
        for (int q = 0; q < CELLS / 4; ++q)
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"((uint32_t)__cvta_generic_to_shared(dst + q * 128)),
                         "l"(src + col0 + 4 * q));
    } else {
#pragma unroll
        for (int k = 0; k < CELLS; ++k) {
            const int c = col0 + k;
            const bool ok = c >= 0 && c < C;
            asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;\n" ::"r"((uint32_t)__cvta_generic_to_shared(ring + pf_off<CELLS>(slot, lane, k))),
                         "l"(ok ? src + c : wall), "r"(ok ? 4 : 0));
        }
    }
    asm volatile("cp.async.commit_group;\n" ::);
}

template <int CELLS, bool EC>
__device__ __forceinline__ void pf_band_body(const int32_t* __restrict__ wall, const int32_t* __restrict__ prev_in,
                                             int32_t* __restrict__ next_out, int32_t* ring, int C, int r0, int h,
                                             int b0, int band_out, int col0, int lane) {
#pragma unroll
    for (int i = 0; i < PfRing<CELLS>::D - 1; ++i)
        if (i < h) pf_issue<CELLS, EC>(ring, wall, r0 + 1 + i, C, col0, lane, i);
        else asm volatile("cp.async.commit_group;\n" ::);
#if __CUDA_ARCH__ >= 900
    cudaGridDependencySynchronize();  // PDL: prev_in is produced by the previous launch
#endif
    int32_t v[CELLS];
    if (!EC && CELLS == 2) {
        const int2 t = *reinterpret_cast<const int2*>(prev_in + col0);
        v[0] = t.x; v[1 % CELLS] = t.y;
    } else if (!EC) {
#pragma unroll
        for (int q = 0; q < CELLS / 4; ++q) {
            const int4 t = *reinterpret_cast<const int4*>(prev_in + col0 + 4 * q);
            v[4 * q] = t.x; v[(4 * q + 1) % CELLS] = t.y; v[(4 * q + 2) % CELLS] = t.z; v[(4 * q + 3) % CELLS] = t.w;
        }
    } else {
#pragma unroll
        for (int k = 0; k < CELLS; ++k) v[k] = (col0 + k >= 0 && col0 + k < C) ? prev_in[col0 + k] : 0;
    }
    for (int i = 0; i < h; ++i) {
        asm volatile("cp.async.wait_group %0;\n" ::"n"(PfRing<CELLS>::D - 2));
        int32_t w[CELLS];
        const int32_t* src = ring + pf_off<CELLS>(i & (PfRing<CELLS>::D - 1), lane, 0);
        if constexpr (CELLS == 2) {
            const int2 t = *reinterpret_cast<const int2*>(src);
            w[0] = t.x; w[1 % CELLS] = t.y;
        }
#pragma unroll
        for (int q = 0; q < CELLS / 4; ++q) {
            const int4 t = reinterpret_cast<const int4*>(src)[q * 32];
            w[4 * q] = t.x; w[(4 * q + 1) % CELLS] = t.y; w[(4 * q + 2) % CELLS] = t.z; w[(4 * q + 3) % CELLS] = t.w;
        }
        if (i + PfRing<CELLS>::D - 1 < h) pf_issue<CELLS, EC>(ring, wall, r0 + i + PfRing<CELLS>::D, C, col0, lane, (i + PfRing<CELLS>::D - 1) & (PfRing<CELLS>::D - 1));
        else asm volatile("cp.async.commit_group;\n" ::);
        const int32_t lnb = __shfl_up_sync(0xffffffffu, v[CELLS - 1], 1);
        const int32_t rnb = __shfl_down_sync(0xffffffffu, v[0], 1);
        int32_t nv[CELLS];
#pragma unroll
        for (int k = 0; k < CELLS; ++k) {
            int32_t l = k > 0 ? v[k > 0 ? k - 1 : 0] : lnb;
            int32_t r = k < CELLS - 1 ? v[k < CELLS - 1 ? k + 1 : 0] : rnb;
            if (EC) {
                const int c = col0 + k;
                if (c <= 0) l = v[k];
                if (c >= C - 1) r = v[k];
            }
            nv[k] = w[k] + min(min(l, v[k]), r);
        }
#pragma unroll
        for (int k = 0; k < CELLS; ++k) v[k] = nv[k];
    }
    asm volatile("cp.async.wait_group 0;\n" ::);
#pragma unroll
    for (int k = 0; k < CELLS; ++k) {
        const int c = col0 + k;
        if (c >= b0 && c < b0 + band_out && c < C) next_out[c] = v[k];
    }
#if __CUDA_ARCH__ >= 900
    cudaTriggerProgrammaticLaunchCompletion();
#endif
}

template <int CELLS>
__global__ void __launch_bounds__(32)
    pf_band(const int32_t* __restrict__ wall, const int32_t* __restrict__ prev_in, int32_t* __restrict__ next_out,
            int R, int C, int r0, int h, int band_out, int vec_ok) {
    __shared__ __align__(16) int32_t ring[PfRing<CELLS>::D * 32 * CELLS];
    const int lane = threadIdx.x;
    const int halo = (h + 3) & ~3;
    const int b0 = blockIdx.x * band_out;
    const int s0 = b0 - halo;
    const int col0 = s0 + lane * CELLS;
    // vector (int2 / int4, cp.async 8/16 B) accesses need C % 4 == 0 and 16-byte aligned wall,
    // prev_in and next_out (vec_ok, checked on the host); otherwise the scalar edge path
    const bool ec = !vec_ok || ((C & 3) != 0) || s0 < 0 || s0 + 32 * CELLS > C;
    if (ec) pf_band_body<CELLS, true>(wall, prev_in, next_out, ring, C, r0, h, b0, band_out, col0, lane);
    else pf_band_body<CELLS, false>(wall, prev_in, next_out, ring, C, r0, h, b0, band_out, col0, lane);
    (void)R;
}

namespace pathfinder {

typedef void (*PfFn)(const int32_t*, const int32_t*, int32_t*, int, int, int, int, int, int);
struct Variant { int cells, mode; PfFn fn; const char* key; };

#define RG_PF(N, M) {N, M, pf_pyramid<N, M>, "void rg::pf_pyramid<" #N ", " #M ">"}
#define RG_PF2(N) RG_PF(N, 0), RG_PF(N, 1)
static const Variant kVariants[] = {
    RG_PF2(1), RG_PF2(2), RG_PF2(3), RG_PF2(4), RG_PF2(5), RG_PF2(6), RG_PF2(7), RG_PF2(8),
    RG_PF2(10), RG_PF2(12), RG_PF2(14), RG_PF2(16), RG_PF2(24), RG_PF2(32),
};
#undef RG_PF2
#undef RG_PF

static const Variant* find(int cells, int mode) {
    for (const auto& v : kVariants)
        if (v.cells == cells && v.mode == mode) return &v;
    return nullptr;
}

struct BandVariant { int cells; PfFn fn; const char* key; };
static const BandVariant kBand[] = {
    {2, pf_band<2>, "void rg::pf_band<2>"},
    {4, pf_band<4>, "void rg::pf_band<4>"},   {8, pf_band<8>, "void rg::pf_band<8>"},
    {16, pf_band<16>, "void rg::pf_band<16>"}, {32, pf_band<32>, "void rg::pf_band<32>"},
};

struct Plan {
    const Variant* v;
    const BandVariant* band;  // warp-band family (flags & RODINIA_STREAM)
    int threads, h, band_out, launches;
};

// Host-only legality (no CUDA call).
rodinia_status plan(const rodinia_granularity& g, int64_t R, int64_t C, Plan* p) {
    if (g.thread_x < 1 || g.thread_y != 1 || g.block_x < 1 || g.block_y != 1 || g.temporal < 1)
        return set_error(RODINIA_E_ILLEGAL_FACTOR, "pathfinder: need thread_x,block_x,temporal >= 1 and "
                                                   "thread_y = block_y = 1 (%s)", gran_str(g).c_str());
    if (g.index_mode != 0 && g.index_mode != 1)
        return set_error(RODINIA_E_ILLEGAL_FACTOR, "pathfinder: index_mode must be 0 or 1");
    const int t = g.thread_x;
    p->band = nullptr;
    if (g.flags & RODINIA_STREAM) {
        if (g.index_mode != 1 || (g.flags & RODINIA_FAITHFUL))
            return set_error(RODINIA_E_NOT_BUILT, "pathfinder: the warp-band family is index_mode 1, non-faithful");
        const int cells = t * g.block_x;
        for (const auto& b : kBand)
            if (b.cells == cells) p->band = &b;
        if (!p->band) return set_error(RODINIA_E_NOT_BUILT, "pathfinder: warp-band with %d cells/lane not built", cells);
        p->v = nullptr;
        p->threads = 32;
        const int64_t steps = R - 1;
        p->h = (int)std::min<int64_t>(g.temporal, std::max<int64_t>(steps, 1));
        const int halo = (p->h + 3) & ~3;
        p->band_out = (32 * cells - 2 * halo) & ~3;
        if (p->band_out < 4)
            return set_error(RODINIA_E_ILLEGAL_FACTOR, "pathfinder: pyramid height %d too large for a %d-column band",
                             p->h, 32 * cells);
        p->launches = steps > 0 ? (int)((steps + p->h - 1) / p->h) : 0;
        return boundary_filter(RODINIA_PATHFINDER, p->band->key, 32, 0, g.flags);
    }
    if ((g.flags & RODINIA_FAITHFUL) && (256 % t != 0))
        return set_error(RODINIA_E_ILLEGAL_FACTOR, "pathfinder: thread factor %d does not divide the "
                                                   "256-thread block (PAPER.md:237)", t);
    const int cells = t * g.block_x;
    p->v = find(cells, g.index_mode);
    if (!p->v) return set_error(RODINIA_E_NOT_BUILT, "pathfinder: %d cells/thread not instantiated", cells);
    int threads = (256 + t - 1) / t;
    threads = ((threads + 31) / 32) * 32;
    if (threads > 1024) threads = 1024;
    p->threads = threads;
    const int64_t steps = R - 1;
    p->h = (int)std::min<int64_t>(g.temporal, std::max<int64_t>(steps, 1));
    p->band_out = threads * cells - 2 * p->h;
    if (p->band_out < 1)
        return set_error(RODINIA_E_ILLEGAL_FACTOR, "pathfinder: pyramid height %d too large for a %d-column "
                                                   "band", p->h, threads * cells);
    p->launches = steps > 0 ? (int)((steps + p->h - 1) / p->h) : 0;
    (void)C;
    return boundary_filter(RODINIA_PATHFINDER, p->v->key, threads, 0, g.flags);
}

rodinia_status run(const int32_t* wall, int32_t* result, int32_t* scratch, int R, int C, const Plan& p,
                   cudaStream_t s) {
    if (p.launches == 0) {
        RG_CUDA(cudaMemcpyAsync(result, wall, (size_t)C * sizeof(int32_t), cudaMemcpyDeviceToDevice, s));
        return RODINIA_OK;
    }
    const int nwarps = p.threads / 32;
    const size_t smem = p.band ? 0 : (size_t)2 * nwarps * 2 * p.v->cells * sizeof(int32_t);
    const int grid = (C + p.band_out - 1) / p.band_out;
    PfFn fn = p.band ? p.band->fn : p.v->fn;
    const int32_t* src = wall;  // row 0 of the wall is the initial cost
    int r0 = 0;
    const int vec_ok = ((reinterpret_cast<uintptr_t>(wall) | reinterpret_cast<uintptr_t>(result) |
                         reinterpret_cast<uintptr_t>(scratch)) % 16) == 0;
    for (int l = 0; l < p.launches; ++l) {
        const int h = std::min(p.h, R - 1 - r0);
        int32_t* dst = ((p.launches - 1 - l) % 2 == 0) ? result : scratch;
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(grid);
        cfg.blockDim = dim3(p.threads);
        cfg.dynamicSmemBytes = smem;
        cfg.stream = s;
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        attr[0].val.programmaticStreamSerializationAllowed = 1;
        cfg.attrs = attr;
        cfg.numAttrs = l > 0 ? 1 : 0;
        RG_CUDA(cudaLaunchKernelEx(&cfg, fn, wall, (const int32_t*)src, dst, R, C, r0, h, p.band_out, vec_ok));
        count_launch();
        src = dst;
        r0 += h;
    }
    return RODINIA_OK;
}

int num_variants() { return (int)(sizeof(kVariants) / sizeof(kVariants[0]) + sizeof(kBand) / sizeof(kBand[0])); }

void variant_info(int i, rodinia_granularity* g, const void** fn, const char** key, int* threads) {
    const int nv = (int)(sizeof(kVariants) / sizeof(kVariants[0]));
    if (i >= nv) {
        const auto& b = kBand[i - nv];
        *g = gran(b.cells, 1, 1, 1, 99, 1, RODINIA_STREAM);
        *fn = (const void*)b.fn;
        *key = b.key;
        *threads = 32;
        return;
    }
    const auto& v = kVariants[i];
    *g = gran(v.cells, 1, 1, 1, 20, v.mode);
    *fn = (const void*)v.fn;
    *key = v.key;
    int t = (256 + v.cells - 1) / v.cells;
    *threads = ((t + 31) / 32) * 32;
}

}  // namespace pathfinder

int pathfinder_num_variants() { return pathfinder::num_variants(); }
void pathfinder_variant_info(int i, rodinia_granularity* g, const void** fn, const char** key, int* threads) {
    pathfinder::variant_info(i, g, fn, key, threads);
}

rodinia_granularity default_gran(rodinia_kernel k, const rodinia_problem& p);
rodinia_status host_buffer(int i, size_t bytes, void** out);
struct HostStage;
HostStage& host_stage();

static rodinia_status pf_validate(const void* wall, const void* result, int64_t R, int64_t C) {
    if (!wall || !result) return set_error(RODINIA_E_INVALID, "pathfinder: null buffer");
    if (R < 1 || C < 1) return set_error(RODINIA_E_INVALID, "pathfinder: rows/cols must be >= 1");
    if (R > (1ll << 31) - 1 || C > (1ll << 31) - 1 || R * C > (1ll << 40))
        return set_error(RODINIA_E_INVALID, "pathfinder: problem too large");
    if (wall == result) return set_error(RODINIA_E_INVALID, "pathfinder: result aliases wall");
    return RODINIA_OK;
}

static rodinia_status pf_resolve(int64_t R, int64_t C, const rodinia_granularity* g, rodinia_granularity* out) {
    if (!gran_is_zero(g)) { *out = *g; return RODINIA_OK; }
    rodinia_problem pb{R, C, 1, 1};
    if (tune_cache_lookup(RODINIA_PATHFINDER, pb, out)) return RODINIA_OK;
    *out = default_gran(RODINIA_PATHFINDER, pb);
    return RODINIA_OK;
}

// Tuner: every instantiated cells/thread x index mode x pyramid height; block factor = 1
// (cells/thread already spans t*b).  Times `reps` batches of 20 calls on synthetic walls.
rodinia_status tune_pathfinder(const rodinia_problem& pr, int reps, rodinia_granularity* best,
                               std::vector<rodinia_tune_row>* rows) {
    const int64_t R = pr.rows, C = pr.cols;
    cudaStream_t s;
    RG_CUDA(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    int32_t *wall = nullptr, *res = nullptr, *scr = nullptr;
    rodinia_status st = RODINIA_OK;
    if (cudaMalloc(&wall, (size_t)R * C * 4) != cudaSuccess || cudaMalloc(&res, (size_t)C * 4) != cudaSuccess ||
        cudaMalloc(&scr, (size_t)C * 4) != cudaSuccess) {
        cudaGetLastError();
        st = set_error(RODINIA_E_NOMEM, "pathfinder tune: allocation failed");
    }
    if (st == RODINIA_OK) cudaMemsetAsync(wall, 3, (size_t)R * C * 4, s);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best_ms = 1e30f;
    const int batch = 20;
    for (int vi = 0; st == RODINIA_OK && vi < pathfinder::num_variants(); ++vi) {
        rodinia_granularity g0;
        const void* fn;
        const char* key;
        int threads;
        pathfinder::variant_info(vi, &g0, &fn, &key, &threads);
        for (int h : {4, 8, 12, 20, 33, 50, 99, 1 << 20}) {
            rodinia_tune_row row;
            memset(&row, 0, sizeof row);
            row.g = gran(g0.thread_x, 1, 1, 1, h, g0.index_mode, g0.flags);
            row.median_ms = -1.f;
            row.model_ms = -1.f;
            pathfinder::Plan p;
            rodinia_status cs = pathfinder::plan(row.g, R, C, &p);
            const PtxasStats* ps = find_stats(key);
            row.regs = ps ? ps->regs : -1;
            row.spill_bytes = ps ? ps->spill_stores + ps->spill_loads : -1;
            row.threads = threads;
            if (cs == RODINIA_OK && p.band) {
                row.smem_bytes = 8 * 32 * p.band->cells * 4;
                row.ctas_per_sm = ctas_per_sm(fn, 32, 0);
                cs = filter_decision(ps, 32, 0, 0);
            } else if (cs == RODINIA_OK) {
                row.smem_bytes = (int)((size_t)2 * (p.threads / 32) * 2 * p.v->cells * 4);
                row.ctas_per_sm = ctas_per_sm(fn, p.threads, row.smem_bytes);
                cs = filter_decision(ps, p.threads, row.smem_bytes, 0);
            }
            if (cs == RODINIA_OK) cs = prune_gate(RODINIA_PATHFINDER, pr, &row);
            if (cs == RODINIA_OK) {
                std::vector<float> ts;
                for (int r = -1; r < reps && cs == RODINIA_OK; ++r) {
                    cudaEventRecord(e0, s);
                    for (int b = 0; b < batch && cs == RODINIA_OK; ++b)
                        cs = pathfinder::run(wall, res, scr, (int)R, (int)C, p, s);
                    cudaEventRecord(e1, s);
                    if (cudaEventSynchronize(e1) != cudaSuccess) {
                        st = cs = cuda_error(cudaGetLastError(), "pathfinder tune", __FILE__, __LINE__);
                    }
                    float ms = 0;
                    cudaEventElapsedTime(&ms, e0, e1);
                    if (r >= 0) ts.push_back(ms / batch);
                }
                if (cs == RODINIA_OK) {
                    std::sort(ts.begin(), ts.end());
                    row.median_ms = ts[ts.size() / 2];
                    if (row.median_ms < best_ms) { best_ms = row.median_ms; *best = row.g; }
                }
            }
            row.status = cs;
            rows->push_back(row);
            if (h >= R - 1) break;  // larger heights are the same plan
        }
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(wall); cudaFree(res); cudaFree(scr);
    cudaStreamDestroy(s);
    if (st == RODINIA_OK && best_ms >= 1e29f) st = set_error(RODINIA_E_FILTERED, "pathfinder tune: no variant survived");
    if (st == RODINIA_OK) tune_cache_store(RODINIA_PATHFINDER, pr, *best, best_ms);
    return st;
}

}  // namespace rg

using namespace rg;

extern "C" rodinia_status rodinia_pathfinder(const int32_t* wall, int64_t R, int64_t C, int32_t* result,
                                             const rodinia_granularity* g, void* stream) {
    RG_TRY(pf_validate(wall, result, R, C));
    rodinia_granularity gg;
    RG_TRY(pf_resolve(R, C, g, &gg));
    pathfinder::Plan p;
    RG_TRY(pathfinder::plan(gg, R, C, &p));
    DeviceInfo di;
    RG_TRY(device_info(&di));
    cudaStream_t s = (cudaStream_t)stream;
    int32_t* scr = nullptr;
    if (p.launches >= 2) RG_TRY(scratch_alloc((void**)&scr, (size_t)C * sizeof(int32_t), s));
    rodinia_status st = pathfinder::run(wall, result, scr, (int)R, (int)C, p, s);
    scratch_free(scr, s);
    return st;
}

extern "C" rodinia_status rodinia_pathfinder_host(const int32_t* wall, int64_t R, int64_t C, int32_t* result,
                                                  const rodinia_granularity* g, void* stream) {
    RG_TRY(pf_validate(wall, result, R, C));
    DeviceInfo di;
    RG_TRY(device_info(&di));
    void *dw, *dr;
    std::lock_guard<std::mutex> lk(host_mutex());  // cached buffers: whole H2D/solve/D2H
    RG_TRY(host_buffer(0, (size_t)R * C * 4, &dw));
    RG_TRY(host_buffer(1, (size_t)C * 4, &dr));
    cudaStream_t s = (cudaStream_t)stream;
    RG_CUDA(cudaMemcpyAsync(dw, wall, (size_t)R * C * 4, cudaMemcpyHostToDevice, s));
    RG_TRY(rodinia_pathfinder((const int32_t*)dw, R, C, (int32_t*)dr, g, stream));
    RG_CUDA(cudaMemcpyAsync(result, dr, (size_t)C * 4, cudaMemcpyDeviceToHost, s));
    RG_CUDA(cudaStreamSynchronize(s));
    return RODINIA_OK;
}

// lud.cu -- granularity-parameterised blocked LU (Rodinia lud) for sm_100a.
//
// Operation: Doolittle LU without pivoting, packed in place (DESIGN.md §3 L1-L6), computed
// with Rodinia's blocked structure.  For panel step k (offset o = P*k):
//   lud_perim     in-tile Doolittle of the P x P diagonal tile (Rodinia's lud_diagonal, done by
//                 warp 0 of every CTA, so no separate launch sits on the chain), then
//                 U12 = L11^-1 A12 (unit-lower forward substitution) for every tile right of
//                 the diagonal, L21 = A21 U11^-1 for every tile below it;
//   lud_internal  A22 -= L21 * U12 for every trailing tile (the paper's "main lud kernel",
//                 PAPER.md:315-353, which its coarsening study targets).
// Granularity (§V) applies to lud_internal: thread coarsening (TX,TY) gives each thread
// TX x TY elements of a tile and shrinks the CTA to (P/TX) x (P/TY) threads; block coarsening
// (bx,by) merges bx x by trailing tiles into one CTA, whose shared memory holds bx U12 tiles
// and by L21 tiles (shared memory x b).  The uncoarsened variant is Rodinia's:
// P = 16, 16 x 16 threads, one element per thread, one tile per CTA.  The per-element
// accumulation order (sum over i ascending, then a -= sum) is the same in every variant, so
// for a fixed panel width every (t, b) variant is bit-identical (reading L5).
//
// lud_diag_final writes the factored diagonal tiles back at the end (and factors the last one).
// The 2*ceil(n/P)-1 launches of one factorisation are captured once into a CUDA graph per
// (device, n, P, granularity) and replayed; kernels read the matrix pointer from a device slot
// the call sets first, so one graph serves every matrix of that size.
#include <cuda_runtime.h>
#include <string.h>
#include <cstdlib>

#include <algorithm>
#include <map>
#include <mutex>
#include <tuple>
#include <vector>

#include "rg_internal.h"
#include "lud_tc.cuh"
#include "workloads.h"

namespace rg {

// ------------------------------------------------------------------ perimeter tiles
// CTA j handles the j-th tile right of the diagonal and the j-th tile below it: lanes 0..P-1
// each own one column of U12 = L11^-1 A12 (forward substitution, unit-lower L11), lanes
// P..2P-1 each own one row of L21 = A21 U11^-1.  Tiles are staged through shared memory with
// coalesced loads, the substitutions run in registers with L11/U11 read by broadcast.
// Threads [0, P) own the U12 columns (unit-lower solve with L11 = dia's strict lower part),
// threads [P, 2P) the L21 rows (solve with U11, then divide by the pivot).  Both are the same
// loop over a row-major matrix M (L11 itself, or U11 transposed) whose rows are read four at a
// time with 128-bit shared loads; per element the subtractions run in ascending j exactly as in
// the two separate loops this replaces (same bits), with half the code (the fully unrolled pair
// of solves overflowed the instruction cache: "no instruction" was the top stall, ncu r02f).
// The diagonal tile of step k (full: only the last tile can be partial, and it has no
// perimeter) is factored by warp 0 of every perimeter CTA itself (diag_factor, the lud_diag
// sequence: same bits), so no separate diagonal launch sits on the chain; A keeps the unfactored
// tile until the end of the factorisation (no later kernel reads it), CTA 0 stores the factored
// tile in dscr[k], and lud_diag_final writes all of them into A (and factors the last tile).
template <int P>
__device__ __forceinline__ void lud_perim_body(float* A, int n, int k, float* __restrict__ dscr) {
    constexpr int LD = P + 4;  // 16-byte aligned rows
    __shared__ __align__(16) float msm[2][P][LD];  // [0]: L11 = dia (row-major), [1]: U11^T
    __shared__ float tile[2][P][P + 1];            // [0]: row tile A12, [1]: column tile A21
    const int o = k * P;
    const int tb = o + P * (blockIdx.x + 1);  // first row/col of this perimeter tile
    const int w = min(P, n - tb);             // its width (last tile may be partial)
    const int tx = threadIdx.x;
    if (tx < 32) {
        float a[P];
        const bool own = tx < P;
#pragma unroll
        for (int j = 0; j < P; ++j) a[j] = own ? A[(size_t)(o + tx) * n + o + j] : 0.f;
        tc::diag_factor<P>(a, P, tx);
        if (own) {
#pragma unroll
            for (int j = 0; j < P; ++j) {
                msm[0][tx][j] = a[j];
                msm[1][j][tx] = a[j];
            }
            if (blockIdx.x == 0) {
#pragma unroll
                for (int j = 0; j < P; ++j) dscr[((size_t)k * P + tx) * P + j] = a[j];
            }
        }
    }
    // fully unrolled: all P loads of a thread are in flight at once (one memory round trip;
    // the rolled loop cost one round trip per iteration, ~16 us per launch at P = 32)
#pragma unroll
    for (int e0 = 0; e0 < P * P; e0 += 2 * P) {
        const int e = e0 + tx, i = e / P, j = e % P;
        tile[0][i][j] = j < w ? A[(size_t)(o + i) * n + tb + j] : 0.f;
        tile[1][i][j] = i < w ? A[(size_t)(tb + i) * n + o + j] : 0.f;
    }
    __syncthreads();
    const int half = tx / P, lane = tx - half * P;  // 0: U12 column `lane`, 1: L21 row `lane`
    const float* M = &msm[half][0][0];
    float v[P];
#pragma unroll
    for (int i = 0; i < P; ++i) v[i] = half == 0 ? tile[0][i][lane] : tile[1][lane][i];
#pragma unroll
    for (int i = 0; i < P; ++i) {
#pragma unroll
        for (int jq = 0; jq < (i + 3) / 4; ++jq) {
            const float4 m = *reinterpret_cast<const float4*>(M + i * LD + 4 * jq);
            const float mm[4] = {m.x, m.y, m.z, m.w};
#pragma unroll
            for (int t = 0; t < 4; ++t)
                if (4 * jq + t < i) v[i] = __fsub_rn(v[i], __fmul_rn(mm[t], v[4 * jq + t < P ? 4 * jq + t : 0]));
        }
        if (half == 1) v[i] = __fdiv_rn(v[i], M[i * LD + i]);
    }
    if (lane < w) {
        if (half == 0) {
#pragma unroll
            for (int i = 0; i < P; ++i) A[(size_t)(o + i) * n + tb + lane] = v[i];
        } else {
#pragma unroll
            for (int i = 0; i < P; ++i) A[(size_t)(tb + lane) * n + o + i] = v[i];
        }
    }
}

template <int P>
__global__ void __launch_bounds__(2 * P) lud_perim(float* const* __restrict__ slot, int n, int k, float* dscr) {
    lud_perim_body<P>(*slot, n, k, dscr);
}

// End of a panel-16/32 factorisation: CTA k < m-1 writes the factored diagonal tile k (dscr)
// into A; CTA m-1 factors the last diagonal tile in A (after the last trailing update).
template <int P>
__global__ void __launch_bounds__(32) lud_diag_final(float* const* __restrict__ slot, int n, const float* __restrict__ dscr) {
    float* A = *slot;
    const int m = (n + P - 1) / P, k = blockIdx.x, o = k * P, lane = threadIdx.x;
    if (k < m - 1) {
        if (lane < P) {
#pragma unroll
            for (int j = 0; j < P; ++j) A[(size_t)(o + lane) * n + o + j] = dscr[((size_t)k * P + lane) * P + j];
        }
        return;
    }
    const int r = min(P, n - o);
    float a[P];
    const bool own = lane < r;
#pragma unroll
    for (int j = 0; j < P; ++j) a[j] = (own && j < r) ? A[(size_t)(o + lane) * n + o + j] : 0.f;
    tc::diag_factor<P>(a, r, lane);
#pragma unroll
    for (int j = 0; j < P; ++j)
        if (own && j < r) A[(size_t)(o + lane) * n + o + j] = a[j];
}


// ------------------------------------------------------------------ trailing update
// The CTA stages by L21 tiles and bx U12 tiles in shared memory and walks its bx*by trailing
// tiles; each thread's TX x TY elements of the next tile are loaded into registers while the
// current tile is being updated (software pipelining of the read-modify-write, which is what
// bounds this kernel by HBM).  MODE 1 with TX % 4 == 0 moves A with 128-bit accesses.
template <int P, int TX, int TY, int MODE>
__device__ __forceinline__ void lud_tile_io(float* A, int n, int cx, int cy, float (&av)[TY][TX], bool load) {
    constexpr int NTX = P / TX, NTY = P / TY;
#pragma unroll
    for (int t_y = 0; t_y < TY; ++t_y) {
        const int ly = MODE == 0 ? (int)threadIdx.y + t_y * NTY : (int)threadIdx.y * TY + t_y;
        const int gr = cy + ly;
        if (MODE == 1 && TX % 4 == 0) {
            const int gc0 = cx + (int)threadIdx.x * TX;
            if (gr < n && gc0 + TX <= n && (n & 3) == 0) {
                float4* p = reinterpret_cast<float4*>(A + (size_t)gr * n + gc0);
#pragma unroll
                for (int q = 0; q < TX / 4; ++q) {
                    if (load) {
                        const float4 t = p[q];
                        av[t_y][4 * q] = t.x; av[t_y][(4 * q + 1) % TX] = t.y;
                        av[t_y][(4 * q + 2) % TX] = t.z; av[t_y][(4 * q + 3) % TX] = t.w;
                    } else {
                        p[q] = make_float4(av[t_y][4 * q], av[t_y][(4 * q + 1) % TX], av[t_y][(4 * q + 2) % TX],
                                           av[t_y][(4 * q + 3) % TX]);
                    }
                }
                continue;
            }
        }
#pragma unroll
        for (int t_x = 0; t_x < TX; ++t_x) {
            const int lx = MODE == 0 ? (int)threadIdx.x + t_x * NTX : (int)threadIdx.x * TX + t_x;
            const int gc = cx + lx;
            if (gr < n && gc < n) {
                if (load) av[t_y][t_x] = A[(size_t)gr * n + gc];
                else A[(size_t)gr * n + gc] = av[t_y][t_x];
            }
        }
    }
}

// register budget: >= 512 resident threads per SM (<= 128 registers per thread)
template <int P, int TX, int TY, int MODE>
__global__ void __launch_bounds__((P / TX) * (P / TY),
                                  (512 / ((P / TX) * (P / TY))) < 32 ? ((512 / ((P / TX) * (P / TY))) > 0 ? (512 / ((P / TX) * (P / TY))) : 1) : 32)
    lud_internal(float* const* __restrict__ slot, int n, int k, int bx, int by) {
    float* A = *slot;
    extern __shared__ __align__(16) float lsm[];
    constexpr int NTX = P / TX, NTY = P / TY, NT = NTX * NTY;
    constexpr int LD = P + 4;  // row pitch of the staged tiles (16-byte aligned rows)
    const int o = k * P;
    const int t0 = o + P;  // first trailing row/col
    const int cx0 = t0 + blockIdx.x * bx * P, cy0 = t0 + blockIdx.y * by * P;
    float* Ush = lsm;                // bx U12 tiles: Ush[(b*P + i)*LD + c] = U12[i][c]
    float* Lsh = lsm + bx * P * LD;  // by L21 tiles, transposed: Lsh[(b*P + i)*LD + r] = L21[r][i]
    const int tid = threadIdx.y * NTX + threadIdx.x;
    float av[TY][TX];
    lud_tile_io<P, TX, TY, MODE>(A, n, cx0, cy0, av, true);  // first tile's A, before staging
    // Stage U12 (row-major, 128-bit) and L21 (transposed) tiles.  Index math uses only the
    // compile-time tile size; the per-tile loops are over the runtime block factors.
    const bool vec = (n & 3) == 0;
    for (int b = 0; b < bx; ++b) {
        const int cb = cx0 + b * P;
        for (int e4 = tid; e4 < P * P / 4; e4 += NT) {
            const int i = e4 / (P / 4), c = 4 * (e4 % (P / 4));
            float4 u = make_float4(0.f, 0.f, 0.f, 0.f);
            const float* src = A + (size_t)(o + i) * n + cb + c;
            if (vec && cb + c + 4 <= n) u = *reinterpret_cast<const float4*>(src);
            else {
                if (cb + c < n) u.x = src[0];
                if (cb + c + 1 < n) u.y = src[1];
                if (cb + c + 2 < n) u.z = src[2];
                if (cb + c + 3 < n) u.w = src[3];
            }
            *reinterpret_cast<float4*>(Ush + (b * P + i) * LD + c) = u;
        }
    }
    for (int b = 0; b < by; ++b) {
        const int rb = cy0 + b * P;
        for (int e4 = tid; e4 < P * P / 4; e4 += NT) {
            const int rr = e4 / (P / 4), i = 4 * (e4 % (P / 4));
            float4 l = make_float4(0.f, 0.f, 0.f, 0.f);
            if (rb + rr < n) {
                const float* src = A + (size_t)(rb + rr) * n + o + i;
                if (vec) l = *reinterpret_cast<const float4*>(src);
                else l = make_float4(src[0], src[1], src[2], src[3]);
            }
            float* d = Lsh + (b * P + i) * LD + rr;
            d[0] = l.x; d[LD] = l.y; d[2 * LD] = l.z; d[3 * LD] = l.w;
        }
    }
    __syncthreads();
    const int ntiles = bx * by;
    for (int t = 0; t < ntiles; ++t) {
        const int b_y = t / bx, b_x = t - b_y * bx;
        float nx[TY][TX];
        if (t + 1 < ntiles) {
            const int n_y = (t + 1) / bx, n_x = (t + 1) - n_y * bx;
            lud_tile_io<P, TX, TY, MODE>(A, n, cx0 + n_x * P, cy0 + n_y * P, nx, true);
        }
        float sum[TY][TX];
#pragma unroll
        for (int t_y = 0; t_y < TY; ++t_y)
#pragma unroll
            for (int t_x = 0; t_x < TX; ++t_x) sum[t_y][t_x] = 0.f;
        const float* Ub = Ush + (b_x * P) * LD;
        const float* Lb = Lsh + (b_y * P) * LD;
#pragma unroll 4
        for (int i = 0; i < P; ++i) {
            float u[TX], l[TY];
            if (MODE == 1 && TX % 4 == 0) {
#pragma unroll
                for (int q = 0; q < TX / 4; ++q) {
                    const float4 t4 = reinterpret_cast<const float4*>(Ub + i * LD + threadIdx.x * TX)[q];
                    u[4 * q] = t4.x; u[(4 * q + 1) % TX] = t4.y; u[(4 * q + 2) % TX] = t4.z; u[(4 * q + 3) % TX] = t4.w;
                }
            } else {
#pragma unroll
                for (int t_x = 0; t_x < TX; ++t_x)
                    u[t_x] = Ub[i * LD + (MODE == 0 ? (int)threadIdx.x + t_x * NTX : (int)threadIdx.x * TX + t_x)];
            }
            if (MODE == 1 && TY % 4 == 0) {
#pragma unroll
                for (int q = 0; q < TY / 4; ++q) {
                    const float4 t4 = reinterpret_cast<const float4*>(Lb + i * LD + threadIdx.y * TY)[q];
                    l[4 * q] = t4.x; l[(4 * q + 1) % TY] = t4.y; l[(4 * q + 2) % TY] = t4.z; l[(4 * q + 3) % TY] = t4.w;
                }
            } else {
#pragma unroll
                for (int t_y = 0; t_y < TY; ++t_y)
                    l[t_y] = Lb[i * LD + (MODE == 0 ? (int)threadIdx.y + t_y * NTY : (int)threadIdx.y * TY + t_y)];
            }
#pragma unroll
            for (int t_y = 0; t_y < TY; ++t_y)
#pragma unroll
                for (int t_x = 0; t_x < TX; ++t_x) sum[t_y][t_x] = __fmaf_rn(l[t_y], u[t_x], sum[t_y][t_x]);
        }
#pragma unroll
        for (int t_y = 0; t_y < TY; ++t_y)
#pragma unroll
            for (int t_x = 0; t_x < TX; ++t_x) av[t_y][t_x] = __fsub_rn(av[t_y][t_x], sum[t_y][t_x]);
        lud_tile_io<P, TX, TY, MODE>(A, n, cx0 + b_x * P, cy0 + b_y * P, av, false);
        if (t + 1 < ntiles) {
#pragma unroll
            for (int t_y = 0; t_y < TY; ++t_y)
#pragma unroll
                for (int t_x = 0; t_x < TX; ++t_x) av[t_y][t_x] = nx[t_y][t_x];
        }
    }
}

// ------------------------------------------------------------------ streaming trailing update
// lud_internal_stream<P,V> (flags RODINIA_STREAM): column-stationary update for B200.  A CTA of
// 256 threads owns 256*V contiguous trailing columns and a chunk of 16*by rows; each thread keeps
// its V columns of U12 (P x V values) in registers, the chunk's L21 rows are staged in shared
// memory (read by broadcast), and A streams through once: one 128-bit load and one store per V
// elements, A rows requested two rows ahead.  Per element the arithmetic is the same sequence as
// every other variant (sum_i l_i u_i ascending with fma, then a -= sum), so results are
// bit-identical for a fixed panel width.  Bound: HBM (8 B per element per step) at P = 16.
#ifndef RG_LUD_RING
#define RG_LUD_RING 8
#endif
constexpr int LUD_RING = RG_LUD_RING;  // rows in flight per thread (cp.async ring depth)
template <int P, int V>
__global__ void __launch_bounds__(256)
    lud_internal_stream(float* const* __restrict__ slot, int n, int k, int chunk_tiles, int unused) {
    float* A = *slot;
    extern __shared__ __align__(16) float Lst[];  // [rows][P]
    (void)unused;
    const int o = k * P, t0 = o + P;
    const int cbase = t0 + blockIdx.x * 256 * V + threadIdx.x * V;
    const int r0 = t0 + blockIdx.y * chunk_tiles * 16;
    const int r1 = min(n, r0 + chunk_tiles * 16);
    if (r0 >= n) return;
    // stage L21 rows of the chunk (row-major P values each)
    for (int e = threadIdx.x; e < (r1 - r0) * P; e += 256) {
        const int rr = e / P, i = e - rr * P;
        Lst[e] = A[(size_t)(r0 + rr) * n + o + i];
    }
    // this thread's U12 columns
    float u[P][V];
    const bool vec = (V % 4 == 0) && ((n & 3) == 0) && cbase + V <= n;
#pragma unroll
    for (int i = 0; i < P; ++i) {
        const float* urow = A + (size_t)(o + i) * n;
        if (vec) {
#pragma unroll
            for (int q = 0; q < V / 4; ++q) {
                const float4 t = *reinterpret_cast<const float4*>(urow + cbase + 4 * q);
                u[i][4 * q] = t.x; u[i][(4 * q + 1) % V] = t.y; u[i][(4 * q + 2) % V] = t.z; u[i][(4 * q + 3) % V] = t.w;
            }
        } else {
#pragma unroll
            for (int v = 0; v < V; ++v) u[i][v] = cbase + v < n ? urow[cbase + v] : 0.f;
        }
    }
    __syncthreads();
    if (cbase >= n) return;
    auto ld = [&](int r, float (&a)[V]) {
        const float* row = A + (size_t)r * n;
        if (vec) {
#pragma unroll
            for (int q = 0; q < V / 4; ++q) {
                const float4 t = *reinterpret_cast<const float4*>(row + cbase + 4 * q);
                a[4 * q] = t.x; a[(4 * q + 1) % V] = t.y; a[(4 * q + 2) % V] = t.z; a[(4 * q + 3) % V] = t.w;
            }
        } else {
#pragma unroll
            for (int v = 0; v < V; ++v) a[v] = cbase + v < n ? row[cbase + v] : 0.f;
        }
    };
    if (vec) {
        // A rows through a per-thread cp.async ring in shared memory (slots [LUD_RING][256][V],
        // thread-private, no barrier): LUD_RING - 1 rows requested ahead of their use
        float* ring = Lst + (((r1 - r0) * P + 3) & ~3);
        const int nrows = r1 - r0;
        auto issue = [&](int rr) {
            if (rr < nrows) {
                const float* src = A + (size_t)(r0 + rr) * n + cbase;
                float* dst = ring + ((rr % LUD_RING) * 256 + threadIdx.x) * V;
#pragma unroll
                for (int q = 0; q < V / 4; ++q)
                    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(
                                     (uint32_t)__cvta_generic_to_shared(dst + 4 * q)),
                                 "l"(src + 4 * q));
            }
            asm volatile("cp.async.commit_group;\n" ::);
        };
#pragma unroll
        for (int rr = 0; rr < LUD_RING - 1; ++rr) issue(rr);
        for (int rr = 0; rr < nrows; ++rr) {
            asm volatile("cp.async.wait_group %0;\n" ::"n"(LUD_RING - 2));  // row rr has landed
            float a[V];
            const float* slotp = ring + ((rr % LUD_RING) * 256 + threadIdx.x) * V;
#pragma unroll
            for (int q = 0; q < V / 4; ++q) {
                const float4 t = reinterpret_cast<const float4*>(slotp)[q];
                a[4 * q] = t.x; a[(4 * q + 1) % V] = t.y; a[(4 * q + 2) % V] = t.z; a[(4 * q + 3) % V] = t.w;
            }
            issue(rr + LUD_RING - 1);  // into the slot read one row ago
            const float* l = Lst + rr * P;
            float sum[V];
#pragma unroll
            for (int v = 0; v < V; ++v) sum[v] = 0.f;
#pragma unroll
            for (int i4 = 0; i4 < P / 4; ++i4) {
                const float4 l4 = reinterpret_cast<const float4*>(l)[i4];
                const float lv[4] = {l4.x, l4.y, l4.z, l4.w};
#pragma unroll
                for (int ii = 0; ii < 4; ++ii)
#pragma unroll
                    for (int v = 0; v < V; ++v) sum[v] = __fmaf_rn(lv[ii], u[4 * i4 + ii][v], sum[v]);
            }
            float* row = A + (size_t)(r0 + rr) * n + cbase;
#pragma unroll
            for (int q = 0; q < V / 4; ++q)
                reinterpret_cast<float4*>(row)[q] =
                    make_float4(__fsub_rn(a[4 * q], sum[4 * q]), __fsub_rn(a[(4 * q + 1) % V], sum[(4 * q + 1) % V]),
                                __fsub_rn(a[(4 * q + 2) % V], sum[(4 * q + 2) % V]),
                                __fsub_rn(a[(4 * q + 3) % V], sum[(4 * q + 3) % V]));
        }
        asm volatile("cp.async.wait_group 0;\n" ::);
        return;
    }
    float a0[V], a1[V];
    ld(r0, a0);
    if (r0 + 1 < r1) ld(r0 + 1, a1);
    for (int r = r0; r < r1; ++r) {
        float a2[V];
        if (r + 2 < r1) ld(r + 2, a2);
        const float* l = Lst + (r - r0) * P;
        float sum[V];
#pragma unroll
        for (int v = 0; v < V; ++v) sum[v] = 0.f;
#pragma unroll
        for (int i4 = 0; i4 < P / 4; ++i4) {
            const float4 l4 = reinterpret_cast<const float4*>(l)[i4];
            const float lv[4] = {l4.x, l4.y, l4.z, l4.w};
#pragma unroll
            for (int ii = 0; ii < 4; ++ii)
#pragma unroll
                for (int v = 0; v < V; ++v) sum[v] = __fmaf_rn(lv[ii], u[4 * i4 + ii][v], sum[v]);
        }
        float res[V];
#pragma unroll
        for (int v = 0; v < V; ++v) res[v] = __fsub_rn(a0[v], sum[v]);
        float* row = A + (size_t)r * n;
        if (vec) {
#pragma unroll
            for (int q = 0; q < V / 4; ++q)
                reinterpret_cast<float4*>(row + cbase)[q] =
                    make_float4(res[4 * q], res[(4 * q + 1) % V], res[(4 * q + 2) % V], res[(4 * q + 3) % V]);
        } else {
#pragma unroll
            for (int v = 0; v < V; ++v)
                if (cbase + v < n) row[cbase + v] = res[v];
        }
#pragma unroll
        for (int v = 0; v < V; ++v) { a0[v] = a1[v]; a1[v] = a2[v]; }
    }
}

namespace tc {
// Launch helper for the captured panel-128 factorisation: every kernel of the latency chain
// (diagonal block, panel solves, next block's update) carries the highest launch priority, so
// that in the graph (instantiated with cudaGraphInstantiateFlagUseNodePriority) it is scheduled
// ahead of the concurrently running remainder update's CTAs.
struct Lnch {
    cudaStream_t s;
    int prio;   // cudaLaunchAttributePriority value (0 = default)
    bool pdl = false;  // programmatic dependent of the previous kernel on the stream
};
template <typename... KArgs, typename... Args>
inline void launch_p(const Lnch& L, void (*fn)(KArgs...), dim3 grid, dim3 block, size_t smem, Args... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = L.s;
    cudaLaunchAttribute at[2];
    int na = 0;
    if (L.prio) {
        at[na].id = cudaLaunchAttributePriority;
        at[na].val.priority = L.prio;
        ++na;
    }
    if (L.pdl) {
        at[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        at[na].val.programmaticStreamSerializationAllowed = 1;
        ++na;
    }
    cfg.attrs = at;
    cfg.numAttrs = na;
    cudaLaunchKernelEx(&cfg, fn, (KArgs)args...);
}

// v3 (round 2): the 1 x 1 case of the 2-D block-cyclic algorithm (ldist, DESIGN.md §5/§6) with
// look-ahead.  Per 128-wide block column k, main branch (high priority): lud_diag128 factors
// A_kk -> lud_trsm128 solves L21 and U12 in one launch, writing the operand images (double-
// buffered by k's parity) -> the rank-128 update of block row / column k+1 (after the previous
// remainder); side branch: the remainder update [e2, n)^2, concurrent with the next block's
// diag/trsm.
// While the trailing matrix is large (remainder update longer than the chain) the block columns
// go in pairs (k, k+1): the main branch updates block rows/columns k+1 AND k+2 with step k's
// panels (a 256-wide band), factors and solves k+1 into chunks 8..15 of the same pair image, and
// updates block row/column k+2 with them; the side branch then applies both steps to
// [e + 256, n)^2 as ONE rank-256 update -- the trailing matrix's read-modify-write (what bounds
// that phase) once per two steps.  pairs_until: pair while n - e >= pairs_until.
// Returns the launch count.
inline int launch_all3(float* const* slot, int n, float* const imgs[4], float* const pimgs[4], float* mimg,
                       cudaStream_t cs, cudaStream_t cs2, cudaEvent_t ev_fork, cudaEvent_t ev_img,
                       cudaEvent_t ev_rest, int prio_hi, int pairs_until) {
    constexpr int NB = ldist::NB;
    int launches = 0;
    cudaEventRecord(ev_fork, cs);
    cudaStreamWaitEvent(cs2, ev_fork, 0);
    const int nb = (n + NB - 1) / NB;
    bool rest_pending = false;
    int pair = 0;
    for (int k = 0; k < nb; ++k) {
        const int o = k * NB, bk = std::min(NB, n - o);
        ldist::diag(slot, (size_t)o * n + o, n, bk, mimg, cs, prio_hi);
        ++launches;
        if (k == nb - 1) break;
        const int e = o + NB, rows = n - e, ng = ldist::img_groups(rows);
        if (pairs_until > 0 && rows >= pairs_until && rows > 3 * NB) {
            // ---- steps k, k+1 as a pair (k+1 < nb - 1: rows > 2 NB)
            float* ia = pimgs[2 * (pair & 1)];
            float* ib = pimgs[2 * (pair & 1) + 1];
            const size_t half = (size_t)16 * ng * tc::KC2 * 8;  // 8 chunks x hi/lo x ng groups
            const ldist::TrsmJob jobs[2] = {{slot, (size_t)e * n + o, n, 1, rows, ia, ng},
                                            {slot, (size_t)o * n + e, n, 0, rows, ib, ng}};
            ldist::trsm(jobs, 2, mimg, cs, prio_hi);
            ++launches;
            if (rest_pending) cudaStreamWaitEvent(cs, ev_rest, 0);
            const int e3 = e + 2 * NB;  // band: block rows / columns k+1, k+2
            const int band[2][4] = {{e, 2 * NB, e, rows}, {e3, n - e3, e, 2 * NB}};
            ldist::update(slot, n, band, 2, e, ia, ng, e, ib, ng, cs, prio_hi);
            ++launches;
            // step k+1
            const int o1 = e, e1 = o1 + NB, rows1 = n - e1;
            ldist::diag(slot, (size_t)o1 * n + o1, n, NB, mimg, cs, prio_hi);
            ++launches;
            const size_t g16 = (size_t)16 * tc::KC2 * 8;  // 128 rows = 16 groups
            const ldist::TrsmJob jobs1[2] = {{slot, (size_t)e1 * n + o1, n, 1, rows1, ia + half + g16, ng},
                                             {slot, (size_t)o1 * n + e1, n, 0, rows1, ib + half + g16, ng}};
            ldist::trsm(jobs1, 2, mimg, cs, prio_hi);
            ++launches;
            cudaEventRecord(ev_img, cs);
            cudaStreamWaitEvent(cs2, ev_img, 0);
            const int e2 = e1 + NB, mb = std::min(NB, n - e1);
            const int next[2][4] = {{e1, rows1, e1, mb}, {e1, mb, e2, n - e2}};  // block column / row k+2
            ldist::update(slot, n, next, 2, e, ia, ng, e, ib, ng, cs, prio_hi, NB, 8);
            ++launches;
            if (e2 < n) {
                const int rest[1][4] = {{e2, n - e2, e2, n - e2}};
                ldist::update(slot, n, rest, 1, e, ia, ng, e, ib, ng, cs2, 0, 2 * NB, 0);
                ++launches;
                cudaEventRecord(ev_rest, cs2);
                rest_pending = true;
            } else {
                rest_pending = false;
            }
            ++pair;
            ++k;  // k+1 done
            continue;
        }
        float* ia = imgs[2 * (k & 1)];
        float* ib = imgs[2 * (k & 1) + 1];
        const ldist::TrsmJob jobs[2] = {{slot, (size_t)e * n + o, n, 1, rows, ia, ng},
                                        {slot, (size_t)o * n + e, n, 0, rows, ib, ng}};
        ldist::trsm(jobs, 2, mimg, cs, prio_hi);
        ++launches;
        cudaEventRecord(ev_img, cs);
        if (rest_pending) cudaStreamWaitEvent(cs, ev_rest, 0);
        cudaStreamWaitEvent(cs2, ev_img, 0);
        const int e2 = std::min(n, e + NB), mb = e2 - e;
        const int next[2][4] = {{e, rows, e, mb}, {e, mb, e2, n - e2}};  // block column / row k+1
        ldist::update(slot, n, next, 2, e, ia, ng, e, ib, ng, cs, prio_hi);
        ++launches;
        if (e2 < n) {
            const int rest[1][4] = {{e2, n - e2, e2, n - e2}};
            ldist::update(slot, n, rest, 1, e, ia, ng, e, ib, ng, cs2, 0);
            ++launches;
            cudaEventRecord(ev_rest, cs2);
            rest_pending = true;
        } else {
            rest_pending = false;
        }
    }
    cudaEventRecord(ev_rest, cs2);
    cudaStreamWaitEvent(cs, ev_rest, 0);  // join
    return launches;
}
}  // namespace tc

__global__ void lud_set_slot(float** slot, float* a) { *slot = a; }

namespace lud {

typedef void (*IntFn)(float* const*, int, int, int, int);
struct Variant { int p, tx, ty, mode; IntFn fn; const char* key; };

#define RG_LI(P, TX, TY, M) {P, TX, TY, M, lud_internal<P, TX, TY, M>, "void rg::lud_internal<" #P ", " #TX ", " #TY ", " #M ">"}
#define RG_LI2(P, TX, TY) RG_LI(P, TX, TY, 0), RG_LI(P, TX, TY, 1)
static const Variant kInternal[] = {
    RG_LI2(16, 1, 1), RG_LI2(16, 2, 1), RG_LI2(16, 1, 2), RG_LI2(16, 2, 2), RG_LI2(16, 4, 1),
    RG_LI2(16, 1, 4), RG_LI2(16, 4, 2), RG_LI2(16, 2, 4), RG_LI2(16, 4, 4), RG_LI2(16, 8, 1),
    RG_LI2(16, 8, 2), RG_LI2(16, 16, 1), RG_LI2(16, 16, 2),
    RG_LI2(32, 1, 1), RG_LI2(32, 2, 1), RG_LI2(32, 2, 2), RG_LI2(32, 4, 1), RG_LI2(32, 4, 2),
    RG_LI2(32, 4, 4), RG_LI2(32, 8, 2), RG_LI2(32, 2, 4), RG_LI2(32, 1, 4), RG_LI2(32, 8, 4),
    RG_LI2(32, 4, 8),
};
#undef RG_LI2
#undef RG_LI

static const Variant* find(int p, int tx, int ty, int mode) {
    for (const auto& v : kInternal)
        if (v.p == p && v.tx == tx && v.ty == ty && v.mode == mode) return &v;
    return nullptr;
}

struct StreamVariant { int p, v; IntFn fn; const char* key; };
static const StreamVariant kStreamInt[] = {
    {16, 4, lud_internal_stream<16, 4>, "void rg::lud_internal_stream<16, 4>"},
    {16, 8, lud_internal_stream<16, 8>, "void rg::lud_internal_stream<16, 8>"},
    {32, 2, lud_internal_stream<32, 2>, "void rg::lud_internal_stream<32, 2>"},
    {32, 4, lud_internal_stream<32, 4>, "void rg::lud_internal_stream<32, 4>"},
};

struct Plan {
    int p;
    bool tc = false;          // panel 128: two-level blocking with the tensor-core trailing update
    const Variant* v;
    const StreamVariant* sv;  // streaming trailing update (flags & RODINIA_STREAM)
    int bx, by;
    size_t smem;
};

rodinia_status plan(const rodinia_granularity& g, int panel, Plan* pl) {
    if (panel == 0) panel = 16;
    if (panel != 16 && panel != 32 && panel != 128)
        return set_error(RODINIA_E_NOT_BUILT, "lud: panel width %d not built (16, 32, 128)", panel);
    if (g.thread_x < 1 || g.thread_y < 1 || g.block_x < 1 || g.block_y < 1 || g.temporal != 1)
        return set_error(RODINIA_E_ILLEGAL_FACTOR, "lud: factors must be >= 1, temporal = 1 (%s)", gran_str(g).c_str());
    pl->tc = false;
    if (panel == 128) {
        // tensor-core path: fixed 128 x 128 MMA tiles; coarsening factors do not apply
        pl->tc = true;
        pl->p = 128;
        pl->v = nullptr;
        pl->sv = nullptr;
        pl->bx = pl->by = 1;
        pl->smem = tc::smem_bytes2();
        return RODINIA_OK;
    }
    if (g.index_mode != 0 && g.index_mode != 1)
        return set_error(RODINIA_E_ILLEGAL_FACTOR, "lud: index_mode must be 0 or 1");
    pl->sv = nullptr;
    if (g.flags & RODINIA_STREAM) {
        if (g.thread_y != 1 || g.index_mode != 1 || (g.flags & RODINIA_FAITHFUL))
            return set_error(RODINIA_E_NOT_BUILT, "lud: stream family needs thread_y = 1, index_mode = 1");
        for (const auto& x : kStreamInt)
            if (x.p == panel && x.v == g.thread_x) pl->sv = &x;
        if (!pl->sv) return set_error(RODINIA_E_NOT_BUILT, "lud: stream variant P=%d V=%d not built", panel, g.thread_x);
        pl->p = panel;
        pl->v = nullptr;
        pl->bx = 1;
        pl->by = g.block_y;  // rows per CTA in 16-row tiles
        // L21 rows of the chunk + the cp.async ring (LUD_RING rows x 256 threads x V)
        pl->smem = (size_t)16 * g.block_y * panel * sizeof(float) + (size_t)LUD_RING * 256 * g.thread_x * sizeof(float);
        if (pl->smem > 227 * 1024) return set_error(RODINIA_E_SMEM, "lud: stream chunk needs %zu B shared memory", pl->smem);
        return boundary_filter(RODINIA_LUD, pl->sv->key, 256, (int)pl->smem, g.flags);
    }
    if (panel % g.thread_x || panel % g.thread_y)
        return set_error(RODINIA_E_ILLEGAL_FACTOR, "lud: thread factors must divide the %dx%d tile (PAPER.md:237)", panel, panel);
    pl->p = panel;
    pl->v = find(panel, g.thread_x, g.thread_y, g.index_mode);
    if (!pl->v) return set_error(RODINIA_E_NOT_BUILT, "lud: internal variant P=%d %s not instantiated", panel, gran_str(g).c_str());
    pl->bx = g.block_x;
    pl->by = g.block_y;
    pl->smem = (size_t)(g.block_x + g.block_y) * panel * (panel + 4) * sizeof(float);
    if (pl->smem > 227 * 1024)
        return set_error(RODINIA_E_SMEM, "lud: block factor (%d,%d) needs %zu B shared memory > 227 KB (PAPER.md:251)",
                         g.block_x, g.block_y, pl->smem);
    return boundary_filter(RODINIA_LUD, pl->v->key, (panel / g.thread_x) * (panel / g.thread_y), (int)pl->smem,
                           g.flags);  // compile-time filter at the boundary
}

typedef void (*PerimFn)(float* const*, int, int, float*);
typedef void (*DiagFinalFn)(float* const*, int, const float*);
static int launch_all(const Plan& pl, float** slot, int n, float* dscr, cudaStream_t s) {
    const int P = pl.p, m = (n + P - 1) / P;
    PerimFn perim = P == 16 ? (PerimFn)lud_perim<16> : (PerimFn)lud_perim<32>;
    DiagFinalFn fin = P == 16 ? (DiagFinalFn)lud_diag_final<16> : (DiagFinalFn)lud_diag_final<32>;
    for (int k = 0; k + 1 < m; ++k) {
        perim<<<m - k - 1, 2 * P, 0, s>>>(slot, n, k, dscr);  // + the diagonal tile of step k
        const int rem = m - k - 1;
        if (pl.sv) {
            const int width = n - P * (k + 1);
            dim3 grid((width + 256 * pl.sv->v - 1) / (256 * pl.sv->v), (width + 16 * pl.by - 1) / (16 * pl.by));
            pl.sv->fn<<<grid, 256, pl.smem, s>>>(slot, n, k, pl.by, 0);
            continue;
        }
        dim3 grid((rem + pl.bx - 1) / pl.bx, (rem + pl.by - 1) / pl.by);
        dim3 block(P / pl.v->tx, P / pl.v->ty);
        pl.v->fn<<<grid, block, pl.smem, s>>>(slot, n, k, pl.bx, pl.by);
    }
    fin<<<m, 32, 0, s>>>(slot, n, dscr);
    return 2 * (m - 1) + 1;
}

// One captured factorisation per (device, n, plan).  The matrix pointer reaches the kernels
// through a device slot written by the graph's own root node (lud_set_slot), whose argument is
// replaced with cudaGraphExecKernelNodeSetParams before every launch.  Launches of one graph
// exec are ordered after each other whatever their streams, and a parameter update only affects
// later launches, so concurrent calls with the same n on different streams each factor their own
// matrix (the slot and the panel-128 operand images are only touched inside the graph).
struct GraphEntry {
    cudaGraph_t graph = nullptr;      // kept alive: `root` must stay a node of it
    cudaGraphExec_t exec = nullptr;
    cudaGraphNode_t root = nullptr;   // the lud_set_slot kernel node
    cudaKernelNodeParams rootp = {};
    float** slot = nullptr;
    float* img = nullptr;   // panel-128 path: the two tensor-core operand images
    float* dscr = nullptr;  // panel 16/32: the factored diagonal tiles (written back at the end)
    int launches = 0;
};
static std::mutex g_mu;
static std::map<std::tuple<int, int, int, int, int, int, int, int, int>, GraphEntry> g_graphs;

rodinia_status run(float* a, int n, const Plan& pl, cudaStream_t s) {
    int dev = 0;
    RG_CUDA(cudaGetDevice(&dev));
    const auto key = pl.tc ? std::make_tuple(dev, n, pl.p, 0, 0, 0, 1, 1, 2)
                   : pl.sv ? std::make_tuple(dev, n, pl.p, pl.sv->v, 0, 1, pl.bx, pl.by, 1)
                           : std::make_tuple(dev, n, pl.p, pl.v->tx, pl.v->ty, pl.v->mode, pl.bx, pl.by, 0);
    std::lock_guard<std::mutex> lk(g_mu);
    GraphEntry& ge = g_graphs[key];
    const int m = (n + pl.p - 1) / pl.p;
    if (!ge.exec) {
        if (!ge.slot) RG_CUDA(cudaMalloc(&ge.slot, sizeof(float*)));
        const void* ifn = pl.tc ? (const void*)tc::lud_tc_update2
                                : pl.sv ? (const void*)pl.sv->fn : (const void*)pl.v->fn;
        const size_t fimg = std::max(tc::img_floats(n), ldist::img_floats(n));
        if (pl.tc && !ge.img)  // 4 operand images + the diagonal-block payload + 4 pair images (v3)
            RG_CUDA(cudaMalloc(&ge.img, (12 * fimg + ldist::mimg_floats()) * sizeof(float)));
        if (!pl.tc && !ge.dscr) RG_CUDA(cudaMalloc(&ge.dscr, (size_t)m * pl.p * pl.p * sizeof(float)));
        if (pl.smem > 48 * 1024)
            RG_CUDA(cudaFuncSetAttribute(ifn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)pl.smem));
        cudaStream_t cs, cs2;
        cudaEvent_t ev[3];
        int prio_lo = 0, prio_hi = 0;
        cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
        // the capture stream carries the high priority (the panel-128 chain's kernel nodes inherit
        // it); the side branch the low one
        RG_CUDA(cudaStreamCreateWithPriority(&cs, cudaStreamNonBlocking, pl.tc ? prio_hi : prio_lo));
        RG_CUDA(cudaStreamCreateWithPriority(&cs2, cudaStreamNonBlocking, prio_lo));
        for (auto& x : ev) RG_CUDA(cudaEventCreateWithFlags(&x, cudaEventDisableTiming));
        cudaGraph_t graph;
        RG_CUDA(cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal));
        lud_set_slot<<<1, 1, 0, cs>>>(ge.slot, a);  // root node; argument replaced per launch
        int nl = 3 * m - 2;
        if (pl.tc) {
            const size_t f = fimg;
            float* const imgs[4] = {ge.img, ge.img + f, ge.img + 2 * f, ge.img + 3 * f};
            float* const pb = ge.img + 4 * f + ldist::mimg_floats();
            float* const pimgs[4] = {pb, pb + 2 * f, pb + 4 * f, pb + 6 * f};
            // pair block columns while the trailing matrix has at least this many rows
            const char* pe = getenv("RG_LUD_PAIR");
            const int pairs_until = pe ? atoi(pe) : n / 2;
            nl = tc::launch_all3(ge.slot, n, imgs, pimgs, ge.img + 4 * f, cs, cs2, ev[0], ev[1], ev[2], prio_hi,
                                 pairs_until);
        } else {
            nl = launch_all(pl, ge.slot, n, ge.dscr, cs);
        }
        cudaError_t e = cudaStreamEndCapture(cs, &graph);
        cudaStreamDestroy(cs);
        cudaStreamDestroy(cs2);
        for (auto& x : ev) cudaEventDestroy(x);
        if (e != cudaSuccess) return cuda_error(e, "lud graph capture", __FILE__, __LINE__);
        size_t nroot = 1;
        cudaGraphNode_t root = nullptr;
        e = cudaGraphGetRootNodes(graph, &root, &nroot);
        if (e == cudaSuccess && nroot == 1) e = cudaGraphKernelNodeGetParams(root, &ge.rootp);
        else if (e == cudaSuccess) e = cudaErrorInvalidValue;
        // per-node launch priorities (the panel-128 chain) only take effect with this flag
        if (e == cudaSuccess) e = cudaGraphInstantiateWithFlags(&ge.exec, graph, cudaGraphInstantiateFlagUseNodePriority);
        if (e != cudaSuccess) {
            ge.exec = nullptr;
            cudaGraphDestroy(graph);
            return cuda_error(e, "lud graph instantiate", __FILE__, __LINE__);
        }
        ge.graph = graph;
        ge.root = root;
        ge.launches = nl;
    }
    void* args[2] = {(void*)&ge.slot, (void*)&a};
    cudaKernelNodeParams kp = ge.rootp;
    kp.kernelParams = args;
    kp.extra = nullptr;
    RG_CUDA(cudaGraphExecKernelNodeSetParams(ge.exec, ge.root, &kp));
    RG_CUDA(cudaGraphLaunch(ge.exec, s));
    count_launch(ge.launches + 1);
    return RODINIA_OK;
}

int num_variants() { return (int)(sizeof(kInternal) / sizeof(kInternal[0]) + sizeof(kStreamInt) / sizeof(kStreamInt[0])); }
void variant_info(int i, rodinia_granularity* g, const void** fn, const char** key, int* threads) {
    const int ni = (int)(sizeof(kInternal) / sizeof(kInternal[0]));
    if (i >= ni) {
        const auto& v = kStreamInt[i - ni];
        *g = gran(v.v, 1, 1, 16, 1, 1, RODINIA_STREAM);
        *fn = (const void*)v.fn;
        *key = v.key;
        *threads = 256;
        return;
    }
    const auto& v = kInternal[i];
    *g = gran(v.tx, v.ty, 1, 1, 1, v.mode);
    *fn = (const void*)v.fn;
    *key = v.key;
    *threads = (v.p / v.tx) * (v.p / v.ty);
}

}  // namespace lud

int lud_num_variants() { return lud::num_variants(); }
void lud_variant_info(int i, rodinia_granularity* g, const void** fn, const char** key, int* threads) {
    lud::variant_info(i, g, fn, key, threads);
}

rodinia_granularity default_gran(rodinia_kernel k, const rodinia_problem& p);
rodinia_status host_buffer(int i, size_t bytes, void** out);

static rodinia_status lud_validate(const void* a, int64_t n, int32_t panel) {
    if (!a) return set_error(RODINIA_E_INVALID, "lud: null buffer");
    if (n < 1 || n > 65535 * 16) return set_error(RODINIA_E_INVALID, "lud: n must be in [1, 1048560]");
    if (panel < 0) return set_error(RODINIA_E_INVALID, "lud: panel < 0");
    return RODINIA_OK;
}

__global__ void lud_fill_k(float* a, int n) {
    // diagonally dominant synthetic matrix for timing (values do not affect the run time)
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < (int64_t)n * n;
         e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = e / n, j = e - i * n;
        uint32_t x = (uint32_t)e * 2654435761u;
        x ^= x >> 13;
        a[e] = (float)(x & 0xffff) * (1.0f / 65536.0f) + (i == j ? (float)n : 0.0f);
    }
}

// Tuner: internal variants of the requested panel width x block factors {1,2,4,7} x {1,2,4}.
// For lud, rodinia_problem.iterations carries the panel width (0 => 16, reading L5).
rodinia_status tune_lud(const rodinia_problem& pr, int reps, rodinia_granularity* best,
                        std::vector<rodinia_tune_row>* rows) {
    const int n = (int)pr.rows;
    const int panel = pr.iterations == 32 ? 32 : 16;
    cudaStream_t s;
    RG_CUDA(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    float* A = nullptr;
    if (cudaMalloc(&A, (size_t)n * n * 4) != cudaSuccess) {
        cudaGetLastError();
        cudaStreamDestroy(s);
        return set_error(RODINIA_E_NOMEM, "lud tune: allocation failed");
    }
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    rodinia_status st = RODINIA_OK;
    float best_ms = 1e30f;
    for (int vi = 0; st == RODINIA_OK && vi < lud::num_variants(); ++vi) {
        rodinia_granularity g0;
        const void* fn;
        const char* key;
        int threads;
        lud::variant_info(vi, &g0, &fn, &key, &threads);
        const int ni = (int)(sizeof(lud::kInternal) / sizeof(lud::kInternal[0]));
        const bool is_stream = vi >= ni;
        if ((is_stream ? lud::kStreamInt[vi - ni].p : lud::kInternal[vi].p) != panel) continue;
        for (int bx : {1, 2, 4, 7})
            for (int by : {1, 2, 4, 8, 16}) {
                if (is_stream ? (bx != 1 || by > 8) : by > 4) continue;  // stream: 16..128-row chunks
                rodinia_tune_row row;
                memset(&row, 0, sizeof row);
                row.g = g0;
                row.g.block_x = bx;
                row.g.block_y = by;
                row.median_ms = -1.f;
                row.model_ms = -1.f;
                lud::Plan pl;
                rodinia_status cs = lud::plan(row.g, panel, &pl);
                const PtxasStats* ps = find_stats(key);
                row.regs = ps ? ps->regs : -1;
                row.spill_bytes = ps ? ps->spill_stores + ps->spill_loads : -1;
                row.threads = threads;
                if (cs == RODINIA_OK) {
                    row.smem_bytes = (int)pl.smem;
                    if (pl.smem > 48 * 1024)
                        cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)pl.smem);
                    row.ctas_per_sm = ctas_per_sm(fn, threads, pl.smem);
                    cs = filter_decision(ps, threads, (int)pl.smem, 0);
                    if (cs == RODINIA_OK && row.ctas_per_sm == 0) cs = RODINIA_E_FILTERED;
                }
                if (cs == RODINIA_OK) cs = prune_gate(RODINIA_LUD, pr, &row);
                if (cs == RODINIA_OK) {
                    std::vector<float> ts;
                    for (int r = -1; r < reps && cs == RODINIA_OK; ++r) {
                        lud_fill_k<<<1184, 256, 0, s>>>(A, n);
                        cudaEventRecord(e0, s);
                        cs = lud::run(A, n, pl, s);
                        cudaEventRecord(e1, s);
                        if (cudaEventSynchronize(e1) != cudaSuccess)
                            st = cs = cuda_error(cudaGetLastError(), "lud tune", __FILE__, __LINE__);
                        float ms = 0;
                        cudaEventElapsedTime(&ms, e0, e1);
                        if (r >= 0) ts.push_back(ms);
                    }
                    if (cs == RODINIA_OK) {
                        std::sort(ts.begin(), ts.end());
                        row.median_ms = ts[ts.size() / 2];
                        if (row.median_ms < best_ms) { best_ms = row.median_ms; *best = row.g; }
                    }
                }
                row.status = cs;
                rows->push_back(row);
            }
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(A);
    cudaStreamDestroy(s);
    if (st == RODINIA_OK && best_ms >= 1e29f) st = set_error(RODINIA_E_FILTERED, "lud tune: no variant survived");
    if (st == RODINIA_OK) tune_cache_store(RODINIA_LUD, pr, *best, best_ms);
    return st;
}

// ================================================================== 2-D block-cyclic distributed LU
// SURVEY §8(f) #3 (the last step: "then a 2-D block-cyclic multi-GPU LU"), DESIGN.md §6.
// Building blocks of rodinia_lud_dist (dist.cu), each acting on one rank's local matrix
// (row-major, leading dimension lda) in NB = 128 blocks:
//   ldist::diag    factor the diagonal block A_kk = L_kk U_kk in place (lud_diag128, one CTA)
//                  and write the images the solves read (U_kk row-major, L_kk transposed,
//                  RN(1/u_jj)), the payload broadcast from the block's owner;
//   ldist::trsm    L_Ik = A_Ik U_kk^-1 (local rows) or U_kJ = L_kk^-1 A_kJ (local columns)
//                  in place, one thread per row / column (lud_trsm128), writing the hi/lo
//                  TF32 operand image of the update as it goes (the payload sent along the
//                  process row / column);
//   ldist::update  the local trailing update A_IJ -= L_Ik U_kJ on the tensor cores
//                  (lud_tc_update2, 3xTF32, the single-GPU panel-128 update kernel).
// Per element the operations and their order depend only on the global element, never on
// the process grid, so every grid gives the same bits (tests/test_gpu_lud_dist.py).
// Doolittle's sequence (reading L5): subtractions in ascending k, L divided by its pivot after
// its k < j terms; products fused (FMA); quotients = IEEE quotients formed from the pivot's
// correctly rounded reciprocal (div_rcp).
constexpr int LD_NB = 128;
constexpr int D128_LD = 140;                   // 16-byte rows; row-per-lane 128-bit reads conflict-free
#ifdef RG_LUD_PROBE  // development timing probes (printf of clock64 phase stamps)
#define LUD_PROBE(i) if (threadIdx.x == 0) pr[i] = clock64()
#define LUD_PROBE_W(i) if (threadIdx.x == 32) pw[i] = clock64()
#else
#define LUD_PROBE(i)
#define LUD_PROBE_W(i)
#endif
// The payload lud_trsm128 reads: U11 and L11^T in a block-upper packed layout (row k of block
// b = k/32 keeps columns [32b, 128): the only ones a solve reads), then RN(1/u_jj).
constexpr int D128_IMG = 32 * (128 + 96 + 64 + 32);  // 10240 floats per packed image
__host__ __device__ constexpr int bup_row(int k) {    // offset of row k's first stored column
    return 4096 * (k >> 5) - 512 * (k >> 5) * ((k >> 5) - 1) + (k & 31) * (128 - 32 * (k >> 5));
}
constexpr size_t d128_mimg_floats() { return (size_t)2 * D128_IMG + 128; }

// RN(a / b) from rb = RN(1 / b) (Markstein): q0 = RN(a rb) lies within one ulp of a/b, the
// residual a - q0 b is exact in one FMA, and RN(q0 + residual * rb) is the correctly rounded
// quotient in the absence of underflow/overflow -- the value __fdiv_rn returns, with the
// reciprocal computed once per pivot.  (b = 0 gives NaN where __fdiv_rn gives inf; zero pivots
// are outside the method, reading L1.)
__device__ __forceinline__ float div_rcp(float a, float b, float rb) {
    const float q0 = __fmul_rn(a, rb);
    const float e = __fmaf_rn(-q0, b, a);
    return __fmaf_rn(e, rb, q0);
}

// Right-looking LU of the rs x rs leading part of a 32 x 32 block held one row per lane
// (a[j] = element (lane, j)), one warp.  Step kk: row kk (final) is broadcast from lane kk,
// lanes kk < i < rs form l_ik = a_ik / u_kk and subtract l_ik u_kj for
// j > kk (others use l = 0: row unchanged).
// rinv[i] = RN(1/u_ii) for i < rs.
// The row is published through the block's own rows in shared memory (sb, row stride ld): lane
// kk stores its row, the warp reads it back as 128-bit broadcasts -- a third of the code of a
// shuffle broadcast, whose per-shuffle convergence fallback ptxas duplicates (the kernel's speed
// depends on instruction fetch).  Lane kk's stored row is final.
__device__ __forceinline__ void diag32_factor(float (&a)[32], int rs, int lane, float* rinv, float* sb, int ld) {
    float myrb = 0.f;
#pragma unroll
    for (int kk = 0; kk < 32; ++kk) {
        if (kk >= rs) break;  // uniform
        float u[32];
        if (lane == kk) {
#pragma unroll
            for (int q = kk / 4; q < 8; ++q)
                *reinterpret_cast<float4*>(sb + kk * ld + 4 * q) = make_float4(a[4 * q], a[4 * q + 1], a[4 * q + 2], a[4 * q + 3]);
        }
        __syncwarp();
#pragma unroll
        for (int q = kk / 4; q < 8; ++q) {  // row kk, broadcast
            const float4 t = *reinterpret_cast<const float4*>(sb + kk * ld + 4 * q);
            u[4 * q] = t.x; u[4 * q + 1] = t.y; u[4 * q + 2] = t.z; u[4 * q + 3] = t.w;
        }
        const float rb = __frcp_rn(u[kk]);
        if (lane == kk) myrb = rb;
        const bool below = lane > kk && lane < rs;
        const float l = below ? div_rcp(a[kk], u[kk], rb) : 0.f;
        a[kk] = below ? l : a[kk];
#pragma unroll
        for (int j = kk + 1; j < 32; ++j) a[j] = __fmaf_rn(-l, u[j], a[j]);
    }
    if (lane < rs) rinv[lane] = myrb;
}

// One CTA of 256 threads factors the r x r block at A (r <= 128, row stride lda) in shared
// memory (rows/columns >= r are zeros and stay zeros), right-looking over 32-wide sub-panels:
// threads 0..95 solve a sub-panel's L rows below the factored diagonal sub-block, threads
// 128..223 its U columns right of it; then warp 0 applies the rank-32 update to the NEXT
// diagonal sub-block and factors it (diag32_factor) while warps 1..7 update the rest of the
// trailing block (4 x 4 register tiles).  Outputs: the block in A, and mimg = [U image |
// L^T image | RN(1/u_jj)] (d128_mimg_floats), written with bulk copies.
__global__ void __launch_bounds__(256, 1) lud_diag128(float* const* __restrict__ slot, size_t off, int lda, int r,
                                                      float* __restrict__ mimg) {
    float* A = *slot + off;  // the matrix pointer comes from a device slot (graph reuse, lud::run)
    constexpr int LD = D128_LD;
    extern __shared__ __align__(128) float S[];  // 132 x LD, then the transposed block T 128 x LD
    __shared__ __align__(16) float rinv[128];
    __shared__ __align__(8) uint64_t mbar;
    float* T = S + 132 * LD;
    // T: the transposed block; the panel solves write their L columns into it as they go (row
    // p+k of T = column p+k of L), so only the diagonal sub-blocks are transposed at the end
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
#ifdef RG_LUD_PROBE
    unsigned long long gt0, gt1, gt2;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt0));
#endif
    asm volatile("griddepcontrol.wait;" ::: "memory");  // (a programmatic dependent on the panel-128 chain)
#ifdef RG_LUD_PROBE
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt1));
    long long pr[16] = {0}, pw[16] = {0};
#endif
    LUD_PROBE(0);
    const bool bulk = r == 128 && (lda & 3) == 0 && ((uintptr_t)A & 15) == 0;
    if (bulk) {  // 128 row copies of 512 B
        if (tid == 0) {
            tc::mbar_init(&mbar, 1);
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
            tc::mbar_expect_tx(&mbar, 128 * 512);
        }
        __syncthreads();
        if (tid < 128) tc::bulk_g2s(S + tid * LD, A + (size_t)tid * lda, 512, &mbar);
    } else {
        float v[64];
#pragma unroll
        for (int q = 0; q < 64; ++q) {
            const int e = tid + 256 * q, i = e >> 7, j = e & 127;
            v[q] = (i < r && j < r) ? A[(size_t)i * lda + j] : 0.f;
        }
#pragma unroll
        for (int q = 0; q < 64; ++q) {
            const int e = tid + 256 * q, i = e >> 7, j = e & 127;
            S[i * LD + j] = v[q];
        }
    }
    constexpr int PADC = LD - 128;
    for (int e = tid; e < 4 * LD + 128 * PADC; e += 256) {  // zero padding: rows 128..131, cols 128..LD-1
        if (e < 4 * LD) S[128 * LD + e] = 0.f;
        else S[((e - 4 * LD) / PADC) * LD + 128 + ((e - 4 * LD) % PADC)] = 0.f;
    }
    if (r < 128)  // columns / rows >= r of T stay zero (the update units reach into them)
        for (int e = tid; e < 128 * LD; e += 256) T[e] = 0.f;
    else
        for (int e = tid; e < 128 * PADC; e += 256) T[(e / PADC) * LD + 128 + (e % PADC)] = 0.f;
    if (bulk) tc::mbar_wait(&mbar, 0);
    __syncthreads();
    LUD_PROBE(1);
    // p = -32 factors the first diagonal sub-block only: one inlined copy of the factorisation
    // (the kernel's speed depends on instruction fetch)
#pragma unroll 1
    for (int p = -32; p + 32 < r; p += 32) {
        const int rest = r - p - 32;  // rows below / columns right of the factored sub-block
        const int nb = p + 32;
        if (p >= 0) {
        if (tid < rest) {
            // L row i: x_j = (a_ij - sum_{k<j} x_k u_kj) / u_jj over the sub-block's columns
            float* xr = S + (p + 32 + tid) * LD + p;
            float x[32];
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                const float4 t = *reinterpret_cast<const float4*>(xr + 4 * q);
                x[4 * q] = t.x; x[4 * q + 1] = t.y; x[4 * q + 2] = t.z; x[4 * q + 3] = t.w;
            }
#pragma unroll
            for (int j = 0; j < 32; ++j) {
                const float* ur = S + (p + j) * LD + p;
                float u[32];
#pragma unroll
                for (int q = j / 4; q < 8; ++q) {
                    const float4 t = *reinterpret_cast<const float4*>(ur + 4 * q);
                    u[4 * q] = t.x; u[4 * q + 1] = t.y; u[4 * q + 2] = t.z; u[4 * q + 3] = t.w;
                }
                x[j] = div_rcp(x[j], u[j], rinv[p + j]);
#pragma unroll
                for (int j2 = j + 1; j2 < 32; ++j2) x[j2] = __fmaf_rn(-x[j], u[j2], x[j2]);
            }
#pragma unroll
            for (int q = 0; q < 8; ++q)
                *reinterpret_cast<float4*>(xr + 4 * q) = make_float4(x[4 * q], x[4 * q + 1], x[4 * q + 2], x[4 * q + 3]);
#pragma unroll
            for (int k = 0; k < 32; ++k) T[(p + k) * LD + p + 32 + tid] = x[k];
        } else if (tid >= 128 && tid - 128 < rest) {
            // U column c: y_i = a_ic - sum_{k<i} l_ik y_k (unit-lower sub-block)
            const int c = p + 32 + (tid - 128);
            float y[32];
#pragma unroll
            for (int i = 0; i < 32; ++i) y[i] = S[(p + i) * LD + c];
#pragma unroll
            for (int k = 0; k < 32; ++k)
#pragma unroll
                for (int i = k + 1; i < 32; ++i) y[i] = __fmaf_rn(-S[(p + i) * LD + p + k], y[k], y[i]);
#pragma unroll
            for (int i = 0; i < 32; ++i) S[(p + i) * LD + c] = y[i];
        }
        __syncthreads();
        LUD_PROBE(3 + 3 * (p / 32));
        {
            // the next diagonal sub-block's rank-32 update first, by all threads (4 elements each)
            const int i = nb + (tid >> 3), j0 = nb + 4 * (tid & 7);
            float4 c = *reinterpret_cast<const float4*>(S + i * LD + j0);
#pragma unroll 8
            for (int k = 0; k < 32; ++k) {
                const float l = -T[(p + k) * LD + i];
                const float4 u = *reinterpret_cast<const float4*>(S + (p + k) * LD + j0);
                c.x = __fmaf_rn(l, u.x, c.x);
                c.y = __fmaf_rn(l, u.y, c.y);
                c.z = __fmaf_rn(l, u.z, c.z);
                c.w = __fmaf_rn(l, u.w, c.w);
            }
            *reinterpret_cast<float4*>(S + i * LD + j0) = c;
        }
        __syncthreads();
        }
        if (warp == 0) {
            // ... then its factorisation, while the other warps update the rest
            float a[32];
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                const float4 c = *reinterpret_cast<const float4*>(S + (nb + lane) * LD + nb + 4 * q);
                a[4 * q] = c.x; a[4 * q + 1] = c.y; a[4 * q + 2] = c.z; a[4 * q + 3] = c.w;
            }
            if (p >= 0) LUD_PROBE(4 + 3 * (p / 32));
            diag32_factor(a, min(32, rest), lane, rinv + nb, S + nb * LD + nb, LD);
#pragma unroll
            for (int q = 0; q < 8; ++q)
                *reinterpret_cast<float4*>(S + (nb + lane) * LD + nb + 4 * q) =
                    make_float4(a[4 * q], a[4 * q + 1], a[4 * q + 2], a[4 * q + 3]);
        } else if (p >= 0) {
            // rank-32 update of the rest of [nb, r)^2: units of 4 rows x 8 columns, consecutive lanes
            // on consecutive row groups of one column group (u rows broadcast, T rows 128-bit);
            // units may reach into the zero padding (rows < 132, columns < LD): 0 - 0 * u
            // warp 4 shares warp 0's scheduler (warp w issues on SMSP w mod 4) and stays out, so the
            // factorisation's dependent chain keeps its issue slots; products on the FP32x2 pipe
            // (FFMA2: element-wise the same RN fused multiply-adds, same bits)
            const int nrg = (rest + 3) / 4, ncg = (rest + 7) / 8;
            const int widx = warp < 4 ? warp - 1 : warp - 2;
            for (int t = warp == 4 ? nrg * ncg : widx * 32 + lane; t < nrg * ncg; t += 192) {
                const int cg = t / nrg, rg = t - cg * nrg;
                if (rg < 8 && cg < 4) continue;  // the next diagonal sub-block (warp 0)
                const int i0 = nb + 4 * rg, j0 = nb + 8 * cg;
                float2 acc[4][4];
#pragma unroll
                for (int a = 0; a < 4; ++a) {
                    const float4 v0 = *reinterpret_cast<const float4*>(S + (i0 + a) * LD + j0);
                    const float4 v1 = *reinterpret_cast<const float4*>(S + (i0 + a) * LD + j0 + 4);
                    acc[a][0] = make_float2(v0.x, v0.y); acc[a][1] = make_float2(v0.z, v0.w);
                    acc[a][2] = make_float2(v1.x, v1.y); acc[a][3] = make_float2(v1.z, v1.w);
                }
#pragma unroll 4
                for (int k = 0; k < 32; ++k) {
                    const float4 u0 = *reinterpret_cast<const float4*>(S + (p + k) * LD + j0);
                    const float4 u1 = *reinterpret_cast<const float4*>(S + (p + k) * LD + j0 + 4);
                    const float4 l4 = *reinterpret_cast<const float4*>(T + (p + k) * LD + i0);
                    const float2 u[4] = {make_float2(u0.x, u0.y), make_float2(u0.z, u0.w), make_float2(u1.x, u1.y),
                                         make_float2(u1.z, u1.w)};
                    const float2 l[4] = {make_float2(-l4.x, -l4.x), make_float2(-l4.y, -l4.y), make_float2(-l4.z, -l4.z),
                                         make_float2(-l4.w, -l4.w)};
#pragma unroll
                    for (int a = 0; a < 4; ++a)
#pragma unroll
                        for (int b = 0; b < 4; ++b) acc[a][b] = __ffma2_rn(l[a], u[b], acc[a][b]);
                }
#pragma unroll
                for (int a = 0; a < 4; ++a) {
                    *reinterpret_cast<float4*>(S + (i0 + a) * LD + j0) = make_float4(acc[a][0].x, acc[a][0].y, acc[a][1].x, acc[a][1].y);
                    *reinterpret_cast<float4*>(S + (i0 + a) * LD + j0 + 4) = make_float4(acc[a][2].x, acc[a][2].y, acc[a][3].x, acc[a][3].y);
                }
            }
            LUD_PROBE_W(p / 32);
        }
        __syncthreads();
        LUD_PROBE(5 + 3 * (p / 32));
    }
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");  // the solves may launch (they wait)
    // outputs: bulk stores of the row-major image, 1/u and the A rows first, then the transposed
    // image built in shared memory meanwhile
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    if (tid == 0)
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(mimg + 2 * D128_IMG),
                     "r"(tc::smem_u32(rinv)), "r"(512u) : "memory");
    if (tid >= 128) {  // packed U image: row k, columns [32b, 128)
        const int k = tid - 128, b = k >> 5;
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(mimg + bup_row(k)),
                     "r"(tc::smem_u32(S + k * LD + 32 * b)), "r"((uint32_t)((128 - 32 * b) * 4)) : "memory");
    }
    if (bulk) {
        if (tid < 128)
            asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], 512;" ::"l"(A + (size_t)tid * lda),
                         "r"(tc::smem_u32(S + tid * LD)) : "memory");
    } else {
        for (int e = tid; e < r * 128; e += 256) {
            const int i = e >> 7, j = e & 127;
            if (j < r) A[(size_t)i * lda + j] = S[i * LD + j];
        }
    }
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    for (int e = tid; e < 4 * 32 * 32; e += 256) {  // the diagonal sub-blocks (U and L parts)
        const int b = e >> 10, i = 32 * b + ((e >> 5) & 31), k = 32 * b + (e & 31);
        T[k * LD + i] = S[i * LD + k];
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    if (tid < 128) {  // packed L^T image
        const int k = tid, b = k >> 5;
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(mimg + D128_IMG + bup_row(k)),
                     "r"(tc::smem_u32(T + k * LD + 32 * b)), "r"((uint32_t)((128 - 32 * b) * 4)) : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    }
    asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // shared memory read before exit
#ifdef RG_LUD_PROBE
    LUD_PROBE(14);
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt2));
    if (tid == 0) printf("diag128 ns: wait %llu body %llu start %llu cyc %lld p0 %lld p1 %lld p2 %lld out %lld\n", gt1 - gt0, gt2 - gt1, gt0,
                         pr[14] - pr[0], pr[5] - pr[2], pr[8] - pr[5], pr[11] - pr[8], pr[14] - pr[11]);
    if (tid == 32) printf("diag128 rest-update end (warp 1): %lld %lld %lld\n", pw[0], pw[1], pw[2]);
    __syncthreads();
    if (tid == 0)
        printf("diag128 r=%d load %lld diag0 %lld | p0 LU %lld dupd %lld factor+rest %lld | p1 %lld %lld %lld | p2 %lld %lld %lld | "
               "out %lld  [p0 start %lld]\n", r, pr[1] - pr[0], pr[2] - pr[1], pr[3] - pr[2], pr[4] - pr[3], pr[5] - pr[4],
               pr[6] - pr[5], pr[7] - pr[6], pr[8] - pr[7], pr[9] - pr[8], pr[10] - pr[9], pr[11] - pr[10],
               pr[14] - pr[11], pr[3]);
#endif
}
constexpr size_t d128_smem() { return (size_t)(132 + 128) * D128_LD * sizeof(float); }

// Triangular solves against the factored 128 x 128 diagonal block (mimg from lud_diag128),
// 64 threads per CTA, one thread per row (lower: L = A U^-1, row t at A + t*lda) or per
// column (upper: U = L^-1 A, column t at A + t, rows at stride lda), `count` of them.  Both are
// the substitution x_j -= sum_{k<j} x_k M[k][j] with M (U, or L transposed) bulk-copied into
// shared memory, in four 32-wide pieces: the solved values of earlier pieces (kept per thread
// in shared memory) are applied first (left-looking, 16 independent FFMA2 chains), then the
// 32-step substitution inside the piece (lower: divided by the pivot after its k < j terms).
// Each solved piece is written to A and, split hi/lo, to the tensor-core operand image `img`
// (ng 8-row groups) of the update, image row = thread index.
constexpr int TR_T = 64, TR_RLD = 129;
constexpr size_t trsm_smem() { return ((size_t)D128_IMG + 128 + (size_t)TR_T * TR_RLD) * sizeof(float); }  // 74.5 KB: 3 CTAs/SM

__device__ __forceinline__ void trsm_load(const float* A, int lda, bool lower, bool vec, bool own, int idx, int c0,
                                          float2 (&x)[16]) {
    if (!own) {
#pragma unroll
        for (int q = 0; q < 16; ++q) x[q] = make_float2(0.f, 0.f);
    } else if (lower && vec) {
        const float4* src = reinterpret_cast<const float4*>(A + (size_t)idx * lda + c0);
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            const float4 t = src[q];
            x[2 * q] = make_float2(t.x, t.y);
            x[2 * q + 1] = make_float2(t.z, t.w);
        }
    } else if (lower) {
#pragma unroll
        for (int q = 0; q < 16; ++q)
            x[q] = make_float2(A[(size_t)idx * lda + c0 + 2 * q], A[(size_t)idx * lda + c0 + 2 * q + 1]);
    } else {
#pragma unroll
        for (int q = 0; q < 16; ++q)
            x[q] = make_float2(A[(size_t)(c0 + 2 * q) * lda + idx], A[(size_t)(c0 + 2 * q + 1) * lda + idx]);
    }
}

// blockIdx.y selects one of (up to) two jobs of one launch (the owner of A_kk solves both its L
// rows and its U columns at once); CTAs past a job's count exit.
struct TrsmJobs {
    ldist::TrsmJob j[2];
};
__global__ void __launch_bounds__(TR_T) lud_trsm128(TrsmJobs jobs, const float* __restrict__ mimg) {
    constexpr int LD = D128_LD;
    extern __shared__ __align__(128) float sm[];
    __shared__ __align__(8) uint64_t mbar;
#ifdef RG_LUD_PROBE
    unsigned long long tg[8];
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tg[0]));
#define TR_PROBE(i) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tg[i]))
#else
#define TR_PROBE(i)
#endif
    asm volatile("griddepcontrol.wait;" ::: "memory");
    TR_PROBE(1);
    const ldist::TrsmJob& jb = jobs.j[blockIdx.y];
    if ((int)blockIdx.x * TR_T >= jb.count) return;
    float* __restrict__ A = *jb.slot + jb.off;
    const int lda = jb.lda, count = jb.count, ng = jb.ng;
    float* __restrict__ img = jb.img;
    float* M = sm;
    float* rinv = sm + D128_IMG;
    float* R = rinv + 128;
    const bool lower = jb.lower != 0;
    const int tid = threadIdx.x, idx = blockIdx.x * TR_T + tid;
    const bool own = idx < count;
    const bool vec = (lda & 3) == 0 && ((uintptr_t)A & 15) == 0;
    if (tid == 0) {  // M and the pivots' reciprocals: two bulk copies
        tc::mbar_init(&mbar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        tc::mbar_expect_tx(&mbar, D128_IMG * 4 + 512);
        tc::bulk_g2s(M, mimg + (lower ? 0 : D128_IMG), D128_IMG * 4, &mbar);
        tc::bulk_g2s(rinv, mimg + 2 * D128_IMG, 512, &mbar);
    }
    float2 x[16], xn[16];
    trsm_load(A, lda, lower, vec, own, idx, 0, x);
    __syncthreads();
    tc::mbar_wait(&mbar, 0);
    TR_PROBE(2);
    float* Rt = R + tid * TR_RLD;
#pragma unroll 1
    for (int p = 0; p < 128; p += 32) {
        if (p + 32 < 128) trsm_load(A, lda, lower, vec, own, idx, p + 32, xn);
        else asm volatile("griddepcontrol.launch_dependents;" ::: "memory");  // last piece
        for (int b = 0; b < p / 32; ++b) {  // the rows of earlier blocks: columns p.. of row k
            const float* mb = M + bup_row(32 * b) + (p - 32 * b);
            const int lb = 128 - 32 * b;
            const float* rb = Rt + 32 * b;
#pragma unroll 4
            for (int kk = 0; kk < 32; ++kk) {
                const float nl = -rb[kk];
                const float2 nl2 = make_float2(nl, nl);
                const float4* mr = reinterpret_cast<const float4*>(mb + kk * lb);
#pragma unroll
                for (int q = 0; q < 8; ++q) {
                    const float4 m = mr[q];
                    x[2 * q] = __ffma2_rn(nl2, make_float2(m.x, m.y), x[2 * q]);
                    x[2 * q + 1] = __ffma2_rn(nl2, make_float2(m.z, m.w), x[2 * q + 1]);
                }
            }
        }
        float xs[32];
#pragma unroll
        for (int q = 0; q < 16; ++q) { xs[2 * q] = x[q].x; xs[2 * q + 1] = x[q].y; }
#pragma unroll
        for (int j = 0; j < 32; ++j) {
            const float4* mr = reinterpret_cast<const float4*>(M + bup_row(p + j));  // columns p..
            float mv[32];
#pragma unroll
            for (int q = j / 4; q < 8; ++q) {
                const float4 m = mr[q];
                mv[4 * q] = m.x; mv[4 * q + 1] = m.y; mv[4 * q + 2] = m.z; mv[4 * q + 3] = m.w;
            }
            if (lower) xs[j] = div_rcp(xs[j], mv[j], rinv[p + j]);
#pragma unroll
            for (int j2 = j + 1; j2 < 32; ++j2) xs[j2] = __fmaf_rn(-xs[j], mv[j2], xs[j2]);
        }
#pragma unroll
        for (int j = 0; j < 32; ++j) Rt[p + j] = xs[j];
        if (own) {
            if (lower && vec) {
#pragma unroll
                for (int q = 0; q < 8; ++q)
                    *reinterpret_cast<float4*>(A + (size_t)idx * lda + p + 4 * q) =
                        make_float4(xs[4 * q], xs[4 * q + 1], xs[4 * q + 2], xs[4 * q + 3]);
            } else if (lower) {
#pragma unroll
                for (int j = 0; j < 32; ++j) A[(size_t)idx * lda + p + j] = xs[j];
            } else {
#pragma unroll
                for (int j = 0; j < 32; ++j) A[(size_t)(p + j) * lda + idx] = xs[j];
            }
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                const float f[4] = {xs[4 * q], xs[4 * q + 1], xs[4 * q + 2], xs[4 * q + 3]};
                tc::img_store4(img, ng, idx, p + 4 * q, f);
            }
        }
#pragma unroll
        for (int q = 0; q < 16; ++q) x[q] = xn[q];
#ifdef RG_LUD_PROBE
        tg[3 + p / 32] = 0;
        TR_PROBE(3 + p / 32);
#endif
    }
#ifdef RG_LUD_PROBE
    if (tid == 0 && blockIdx.x == 0 && blockIdx.y == 0)
        printf("trsm ns: count %d wait %llu mbar %llu p0 %llu p1 %llu p2 %llu p3 %llu start %llu\n", count, tg[1] - tg[0],
               tg[2] - tg[1], tg[3] - tg[2], tg[4] - tg[3], tg[5] - tg[4], tg[6] - tg[5], tg[0]);
#endif
}
#undef TR_PROBE

namespace ldist {
size_t mimg_floats() { return d128_mimg_floats(); }
// padded to whole 256-wide tiles plus one spare (the update's 128 x 256 tiles read B columns
// up to the next multiple of 256 past the rectangle's start)
int img_groups(int64_t rows) { return (int)(((rows + 255) / 256 + 1) * 32); }
size_t img_floats(int64_t rows) { return (size_t)16 * img_groups(rows) * tc::KC2 * 8; }

rodinia_status diag(float* const* slot, size_t off, int lda, int r, float* mimg, cudaStream_t s, int prio) {
    static bool attr = false;
    if (!attr) {
        RG_CUDA(cudaFuncSetAttribute((const void*)lud_diag128, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)d128_smem()));
        attr = true;
    }
    tc::launch_p(tc::Lnch{s, prio, prio != 0}, lud_diag128, dim3(1), dim3(256), d128_smem(), slot, off, lda, r, mimg);
    RG_CUDA(cudaGetLastError());
    count_launch();
    return RODINIA_OK;
}

rodinia_status trsm(const TrsmJob* job, int njobs, const float* mimg, cudaStream_t s, int prio) {
    static bool attr = false;
    if (!attr) {
        RG_CUDA(cudaFuncSetAttribute((const void*)lud_trsm128, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)trsm_smem()));
        attr = true;
    }
    TrsmJobs js;
    memset(&js, 0, sizeof js);
    int nj = 0, cmax = 0;
    for (int i = 0; i < njobs && i < 2; ++i)
        if (job[i].count > 0) {
            js.j[nj++] = job[i];
            cmax = std::max(cmax, job[i].count);
        }
    if (nj == 0) return RODINIA_OK;
    tc::launch_p(tc::Lnch{s, prio, prio != 0}, lud_trsm128, dim3((cmax + TR_T - 1) / TR_T, nj), dim3(TR_T), trsm_smem(), js, mimg);
    RG_CUDA(cudaGetLastError());
    count_launch();
    return RODINIA_OK;
}

rodinia_status set_slot(float** slot, float* a, cudaStream_t s) {
    lud_set_slot<<<1, 1, 0, s>>>(slot, a);
    RG_CUDA(cudaGetLastError());
    return RODINIA_OK;
}

rodinia_status update(float* const* slot, int lda, const int (*rect)[4], int nr, int a_base, const float* ia,
                      int nga, int b_base, const float* ib, int ngb, cudaStream_t s, int prio, int kk, int c0) {
    static bool attr = false;
    if (!attr) {
        RG_CUDA(cudaFuncSetAttribute((const void*)tc::lud_tc_update3<64>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)tc::Upd3<64>::smem()));
        RG_CUDA(cudaFuncSetAttribute((const void*)tc::lud_tc_update3<128>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)tc::Upd3<128>::smem()));
        RG_CUDA(cudaFuncSetAttribute((const void*)tc::lud_tc_update3<256>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)tc::Upd3<256>::smem()));
        attr = true;
    }
    // 128 x 256 C tiles when every rectangle is wider than 128 columns (the remainder update),
    // else 128 x 128 (block column k+1 is exactly 128 wide)
    bool wide = true;
    int live = 0;
    for (int i = 0; i < nr && i < 2; ++i)
        if (rect[i][1] > 0 && rect[i][3] > 0) {
            ++live;
            wide = wide && rect[i][3] > 128;
        }
    if (live == 0) return RODINIA_OK;
    // the thin next-block update (on the factorisation's critical chain): 128 x 64 tiles, twice
    // as many CTAs of half the work
    // (the 256-wide band of a block-column pair is on the chain too: narrow tiles there as well)
    if (prio != 0) wide = false;
    const int bn = wide ? 256 : 64;
    tc::Args a;
    a.nrect = 0;
    for (int i = 0; i < nr && i < 2; ++i)  // rect[i] = {r0, m, c0, nn}
        if (rect[i][1] > 0 && rect[i][3] > 0)
            a.rect[a.nrect++] = tc::make_rect(rect[i][0], rect[i][2], rect[i][1], rect[i][3], 0, kk, bn);
    if (a.nrect == 1) a.rect[1] = a.rect[0];
    const tc::Img im{ia, ib, a_base, b_base, nga, ngb, c0};
    const int grid = a.rect[0].tiles + (a.nrect == 2 ? a.rect[1].tiles : 0);
    if (wide)
        tc::launch_p(tc::Lnch{s, prio, prio != 0}, tc::lud_tc_update3<256>, dim3(grid), dim3(128), tc::Upd3<256>::smem(), slot, lda, a, im);
    else
        tc::launch_p(tc::Lnch{s, prio, prio != 0}, tc::lud_tc_update3<64>, dim3(grid), dim3(128), tc::Upd3<64>::smem(), slot, lda, a, im);
    RG_CUDA(cudaGetLastError());
    count_launch();
    return RODINIA_OK;
}
}  // namespace ldist

}  // namespace rg

using namespace rg;

extern "C" rodinia_status rodinia_lud(float* a, int64_t n, int32_t panel, const rodinia_granularity* g, void* stream) {
    RG_TRY(lud_validate(a, n, panel));
    rodinia_granularity gg;
    if (!gran_is_zero(g)) gg = *g;
    else {
        rodinia_problem pb{n, n, panel == 32 ? 32 : 16, 1};
        if (!tune_cache_lookup(RODINIA_LUD, pb, &gg)) gg = default_gran(RODINIA_LUD, pb);
    }
    lud::Plan pl;
    RG_TRY(lud::plan(gg, panel, &pl));
    DeviceInfo di;
    RG_TRY(device_info(&di));
    cudaStream_t s = (cudaStream_t)stream;
    if ((reinterpret_cast<uintptr_t>(a) & 15) == 0) return lud::run(a, (int)n, pl, s);
    // The kernels' 128-bit accesses (and the panel-128 bulk reduce-add) need a 16-byte aligned
    // matrix; an offset view is factored in an aligned stream-ordered copy (same kernels, same
    // bits) and copied back.
    const size_t bytes = (size_t)n * n * sizeof(float);
    float* t = nullptr;
    RG_TRY(scratch_alloc((void**)&t, bytes, s));
    rodinia_status st = RODINIA_OK;
    if (cudaMemcpyAsync(t, a, bytes, cudaMemcpyDeviceToDevice, s) != cudaSuccess)
        st = cuda_error(cudaGetLastError(), "lud aligned copy", __FILE__, __LINE__);
    if (st == RODINIA_OK) st = lud::run(t, (int)n, pl, s);
    if (st == RODINIA_OK && cudaMemcpyAsync(a, t, bytes, cudaMemcpyDeviceToDevice, s) != cudaSuccess)
        st = cuda_error(cudaGetLastError(), "lud aligned copy", __FILE__, __LINE__);
    scratch_free(t, s);
    return st;
}

extern "C" rodinia_status rodinia_lud_host(float* a, int64_t n, int32_t panel, const rodinia_granularity* g,
                                           void* stream) {
    RG_TRY(lud_validate(a, n, panel));
    DeviceInfo di;
    RG_TRY(device_info(&di));
    void* da;
    std::lock_guard<std::mutex> lk(host_mutex());  // cached buffers: whole H2D/solve/D2H
    RG_TRY(host_buffer(0, (size_t)n * n * 4, &da));
    cudaStream_t s = (cudaStream_t)stream;
    RG_CUDA(cudaMemcpyAsync(da, a, (size_t)n * n * 4, cudaMemcpyHostToDevice, s));
    RG_TRY(rodinia_lud((float*)da, n, panel, g, stream));
    RG_CUDA(cudaMemcpyAsync(a, da, (size_t)n * n * 4, cudaMemcpyDeviceToHost, s));
    RG_CUDA(cudaStreamSynchronize(s));
    return RODINIA_OK;
}

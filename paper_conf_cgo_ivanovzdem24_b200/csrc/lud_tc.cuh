// lud_tc.cuh -- tensor-core (tcgen05, kind::tf32, 3xTF32) rank-K update C -= A*B for the
// panel-128 lud path.  Self-contained (CUDA runtime only) so a standalone layout test can
// include it; lud.cu includes it inside namespace rg.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <algorithm>

namespace rg {
// ------------------------------------------------------------------ tensor-core trailing update
// Panel width 128 (DESIGN.md §5 "lud on tensor cores").  Two-level blocking:
// every 128-wide outer block runs the panel-32 steps (lud_diag<32>, lud_perim<32>) with their
// rank-32 updates restricted to the outer block's L-shaped panel region, then ONE rank-128
// update of the trailing matrix A22 -= L21 * U12 on the 5th-generation tensor cores
// (tcgen05.mma kind::tf32, accumulator in TMEM).  fp32 accuracy comes from the 3xTF32 split:
// x = hi + lo with hi = x with its 13 low mantissa bits cleared (exactly a TF32 value) and
// lo = x - hi (exact in fp32); A*B ~ hi*hi + hi*lo + lo*hi, dropping lo*lo (relative 2^-22)
// and the TF32 truncation of lo (relative 2^-21).  The inner rank-32 updates use the same
// kernel with K = 32.
//
// lud_tc_update: one 128 x 128 tile of C per CTA, 128 threads.  K is processed in chunks of KC:
// all threads stage the chunk's A (128 x KC) and B^T (128 x KC) hi/lo parts, both as K-major
// core matrices, into a double-buffered shared-memory stage, one
// thread issues 3 * KC/8 tcgen05.mma and commits them to the stage's mbarrier; the epilogue
// reads the accumulator with tcgen05.ld (warp w owns TMEM lanes 32w..32w+31 = tile rows) and
// does C -= acc in place.  No-swizzle canonical layouts (cute/atom/mma_traits_sm100.hpp):
//   K-major  ((8,m),2):((16B,SBO),LBO)   : 8-row x 16-byte core matrices, LBO = K step
namespace tc {
constexpr int BM = 128, BN = 128;

struct Rect {
    int r0, c0, m, nn;   // C rows [r0, r0+m), cols [c0, c0+nn)
    int k0, kk;          // A = rows r0.. x cols [k0, k0+kk);  B = rows [k0, k0+kk) x cols c0..
    int tiles_x, tiles;  // tile grid of this rectangle
};
struct Args {
    Rect rect[2];
    int nrect;
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint64_t sm_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    uint64_t d = (uint64_t)((saddr >> 4) & 0x3FFFu);
    d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
    d |= (uint64_t)1 << 46;  // descriptor version (sm_100); base offset 0, SWIZZLE_NONE
    return d;
}

// kind::tf32, D f32, A and B K-major, M = 128, N = 128
constexpr uint32_t kIdesc = (1u << 4) | (2u << 7) | (2u << 10) | (0u << 15) | (0u << 16) |
                            ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);

__device__ __forceinline__ void mma_tf32(uint32_t tmem, uint64_t ad, uint64_t bd, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(tmem),
        "l"(ad), "l"(bd), "r"(kIdesc), "r"(acc));
}

__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count));
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred P1;\n\t"
        "LAB_WAIT:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
        "@P1 bra DONE;\n\t"
        "bra LAB_WAIT;\n\t"
        "DONE:\n\t}\n" ::"r"(smem_u32(b)),
        "r"(parity));
}

__device__ __forceinline__ void split_tf32(float x, float& hi, float& lo) {
    hi = __uint_as_float(__float_as_uint(x) & 0xFFFFE000u);
    lo = __fsub_rn(x, hi);
}

template <int KC>
__global__ void __launch_bounds__(128) lud_tc_update(float* const* __restrict__ slot, int n, Args args) {
    constexpr int PART = BM * KC * 4;              // bytes of one operand part (hi or lo)
    constexpr int STAGE = 4 * PART;                // A hi, A lo, B hi, B lo
    constexpr uint32_t SBO_A = (KC / 4) * 128;     // K-major: 8-row groups
    extern __shared__ __align__(1024) uint8_t sm[];
    uint64_t* mbar = reinterpret_cast<uint64_t*>(sm + 2 * STAGE);
    uint32_t* tslot = reinterpret_cast<uint32_t*>(mbar + 2);
    float* A = *slot;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;

    int b = blockIdx.x, ri = 0;
    if (args.nrect == 2 && b >= args.rect[0].tiles) { b -= args.rect[0].tiles; ri = 1; }
    const Rect rc = ri ? args.rect[1] : args.rect[0];
    const int ty = b / rc.tiles_x, tx = b - ty * rc.tiles_x;
    const int row0 = rc.r0 + ty * BM, col0 = rc.c0 + tx * BN;
    const int rend = rc.r0 + rc.m, cend = rc.c0 + rc.nn, kend = rc.k0 + rc.kk;
    const bool vec = (n & 3) == 0;

    if (tid == 0) {
        mbar_init(&mbar[0], 1);
        mbar_init(&mbar[1], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" ::"r"(smem_u32(tslot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = *tslot;

    const int nchunks = (rc.kk + KC - 1) / KC;
    for (int c = 0; c < nchunks; ++c) {
        const int s = c & 1;
        if (c >= 2) mbar_wait(&mbar[s], ((c - 2) >> 1) & 1);  // MMAs of chunk c-2 released stage s
        uint8_t* st = sm + s * STAGE;
        const int kc0 = rc.k0 + c * KC;
        // A: 128 rows x KC (K contiguous in A), K-major core matrices
        for (int e = tid; e < BM * KC / 4; e += 128) {
            const int rr = e & 7, kq = (e >> 3) % (KC / 4), g = (e >> 3) / (KC / 4);
            const int r = row0 + g * 8 + rr, k = kc0 + 4 * kq;
            float v[4] = {0.f, 0.f, 0.f, 0.f};
            if (r < rend) {
                const float* src = A + (size_t)r * n + k;
                if (vec && k + 4 <= kend) {
                    const float4 t = *reinterpret_cast<const float4*>(src);
                    v[0] = t.x; v[1] = t.y; v[2] = t.z; v[3] = t.w;
                } else {
#pragma unroll
                    for (int q = 0; q < 4; ++q) v[q] = k + q < kend ? src[q] : 0.f;
                }
            }
            float4 h, l;
            split_tf32(v[0], h.x, l.x); split_tf32(v[1], h.y, l.y);
            split_tf32(v[2], h.z, l.z); split_tf32(v[3], h.w, l.w);
            const int off = g * SBO_A + kq * 128 + rr * 16;
            *reinterpret_cast<float4*>(st + off) = h;
            *reinterpret_cast<float4*>(st + PART + off) = l;
        }
        // B: KC rows x 128 columns (N contiguous in A), stored transposed as K-major core
        // matrices (kind::tf32 reads MN-major B as zeros on this part; probed).  A thread
        // gathers 4 consecutive k of one column (4 warp-coalesced scalar loads) and writes them
        // as one 16-byte chunk; the 8 threads of a store phase hold 8 consecutive columns, i.e.
        // 128 contiguous bytes of one core matrix (no bank conflicts).
        for (int e = tid; e < BN * KC / 4; e += 128) {
            const int jj = e % BN, kq = e / BN;
            const int j = col0 + jj, k = kc0 + 4 * kq;
            float v[4] = {0.f, 0.f, 0.f, 0.f};
            if (j < cend) {
#pragma unroll
                for (int q = 0; q < 4; ++q) v[q] = k + q < kend ? A[(size_t)(k + q) * n + j] : 0.f;
            }
            float4 h, l;
            split_tf32(v[0], h.x, l.x); split_tf32(v[1], h.y, l.y);
            split_tf32(v[2], h.z, l.z); split_tf32(v[3], h.w, l.w);
            const int off = (jj >> 3) * SBO_A + kq * 128 + (jj & 7) * 16;
            *reinterpret_cast<float4*>(st + 2 * PART + off) = h;
            *reinterpret_cast<float4*>(st + 3 * PART + off) = l;
        }
        // generic-proxy smem writes -> visible to the tensor core (async proxy)
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncthreads();
        if (tid == 0) {
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            const uint32_t a_hi = smem_u32(st), a_lo = a_hi + PART, b_hi = a_hi + 2 * PART, b_lo = a_hi + 3 * PART;
#pragma unroll
            for (int ks = 0; ks < KC / 8; ++ks) {
                const uint64_t adh = sm_desc(a_hi + ks * 256, 128, SBO_A), adl = sm_desc(a_lo + ks * 256, 128, SBO_A);
                const uint64_t bdh = sm_desc(b_hi + ks * 256, 128, SBO_A), bdl = sm_desc(b_lo + ks * 256, 128, SBO_A);
                mma_tf32(tmem, adl, bdh, (c | ks) != 0);
                mma_tf32(tmem, adh, bdl, 1);
                mma_tf32(tmem, adh, bdh, 1);
            }
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                             smem_u32(&mbar[s]))
                         : "memory");
        }
    }
    mbar_wait(&mbar[(nchunks - 1) & 1], ((nchunks - 1) >> 1) & 1);
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");

    // epilogue: warp w reads TMEM lanes 32w.. (tile rows), 32 columns per load
    const int r = row0 + warp * 32 + lane;
#pragma unroll 1
    for (int jb = 0; jb < BN / 32; ++jb) {
        uint32_t v[32];
        const uint32_t taddr = tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)(jb * 32);
        asm volatile(
            "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
            "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
            : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
              "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]),
              "=r"(v[15]), "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]),
              "=r"(v[22]), "=r"(v[23]), "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]),
              "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
            : "r"(taddr));
        // the wait carries v[] as operands so no use of them can be scheduled before it
        asm volatile("tcgen05.wait::ld.sync.aligned;"
                     : "+r"(v[0]), "+r"(v[1]), "+r"(v[2]), "+r"(v[3]), "+r"(v[4]), "+r"(v[5]), "+r"(v[6]),
                       "+r"(v[7]), "+r"(v[8]), "+r"(v[9]), "+r"(v[10]), "+r"(v[11]), "+r"(v[12]), "+r"(v[13]),
                       "+r"(v[14]), "+r"(v[15]), "+r"(v[16]), "+r"(v[17]), "+r"(v[18]), "+r"(v[19]),
                       "+r"(v[20]), "+r"(v[21]), "+r"(v[22]), "+r"(v[23]), "+r"(v[24]), "+r"(v[25]),
                       "+r"(v[26]), "+r"(v[27]), "+r"(v[28]), "+r"(v[29]), "+r"(v[30]), "+r"(v[31])
                     :
                     : "memory");
        if (r < rend) {
            float* crow = A + (size_t)r * n;
            const int cb = col0 + jb * 32;
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                const int cc = cb + 4 * q;
                if (vec && cc + 4 <= cend) {
                    float4 t = *reinterpret_cast<float4*>(crow + cc);
                    t.x = __fsub_rn(t.x, __uint_as_float(v[4 * q]));
                    t.y = __fsub_rn(t.y, __uint_as_float(v[4 * q + 1]));
                    t.z = __fsub_rn(t.z, __uint_as_float(v[4 * q + 2]));
                    t.w = __fsub_rn(t.w, __uint_as_float(v[4 * q + 3]));
                    *reinterpret_cast<float4*>(crow + cc) = t;
                } else {
#pragma unroll
                    for (int e = 0; e < 4; ++e)
                        if (cc + e < cend) crow[cc + e] = __fsub_rn(crow[cc + e], __uint_as_float(v[4 * q + e]));
                }
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" ::"r"(tmem));
}

#ifndef RG_LUD_KC
#define RG_LUD_KC 16
#endif
constexpr int KC_MAIN = RG_LUD_KC;  // K chunk per stage: 16 -> 64 KB smem, 3 CTAs per SM
constexpr size_t smem_bytes(int kc) { return (size_t)2 * 4 * BM * kc * 4 + 64; }

inline Rect make_rect(int r0, int c0, int m, int nn, int k0, int kk) {
    Rect r;
    r.r0 = r0; r.c0 = c0; r.m = m; r.nn = nn; r.k0 = k0; r.kk = kk;
    r.tiles_x = (nn + BN - 1) / BN;
    r.tiles = r.tiles_x * ((m + BM - 1) / BM);
    return r;
}

// C -= A*B over one or two rectangles (skipped when empty)
inline void launch_update(float* const* slot, int n, const Rect* rs, int nr, cudaStream_t s) {
    Args a;
    a.nrect = 0;
    for (int i = 0; i < nr; ++i)
        if (rs[i].m > 0 && rs[i].nn > 0 && rs[i].kk > 0) a.rect[a.nrect++] = rs[i];
    if (a.nrect == 0) return;
    if (a.nrect == 1) a.rect[1] = a.rect[0];
    const int grid = a.rect[0].tiles + (a.nrect == 2 ? a.rect[1].tiles : 0);
    lud_tc_update<KC_MAIN><<<grid, 128, smem_bytes(KC_MAIN), s>>>(slot, n, a);
}

}  // namespace tc
}  // namespace rg

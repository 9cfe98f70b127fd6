// lud_tc.cuh -- tensor-core (tcgen05, kind::tf32, 3xTF32) rank-K update C -= A*B for the
// panel-128 lud path.  Self-contained (CUDA runtime only) so a standalone layout test can
// include it; lud.cu includes it inside namespace rg.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <algorithm>

namespace rg {
// ------------------------------------------------------------------ tensor-core trailing update
// Panel width 128 (DESIGN.md §5 "lud on tensor cores"): per 128-wide block
// column, the diagonal block and the L21 / U12 panels are factored / solved by lud_diag128 and
// lud_trsm128 (lud.cu), then ONE rank-128 update of the trailing matrix A22 -= L21 * U12 runs
// on the 5th-generation tensor cores (tcgen05.mma kind::tf32, accumulator in TMEM).  fp32
// accuracy comes from the 3xTF32 split: x = hi + lo with hi = x with its 13 low mantissa bits
// cleared (exactly a TF32 value) and lo = x - hi (exact in fp32); A*B ~ hi*hi + hi*lo + lo*hi,
// dropping lo*lo (relative 2^-22) and the TF32 truncation of lo (relative 2^-21).
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

// In-tile Doolittle of a P x P diagonal tile held one row per lane (a[j] = element (lane, j);
// rows/columns >= r are ignored): step kk broadcasts row kk with warp shuffles and every lane
// below it subtracts l_ik * u_kj.  Per element this is Doolittle's sequence (products
// subtracted in ascending k, L divided by the pivot after its k < j terms) with separate
// multiply and subtract as in Rodinia's lud_diagonal.  lud_diag and the panel-128 update's
// fused diagonal both call this, so both give the same bits.
template <int P>
__device__ __forceinline__ void diag_factor(float (&a)[P], int r, int lane) {
    const bool own = lane < r;
#pragma unroll
    for (int kk = 0; kk < P - 1; ++kk) {
        if (kk >= r - 1) break;  // uniform
        const float piv = __shfl_sync(0xffffffffu, a[kk], kk);
        const bool below = lane > kk && own;
        const float l = __fdiv_rn(a[kk], piv);
        if (below) a[kk] = l;
#pragma unroll
        for (int j = kk + 1; j < P; ++j) {
            const float ukj = __shfl_sync(0xffffffffu, a[j], kk);
            if (below) a[j] = __fsub_rn(a[j], __fmul_rn(l, ukj));
        }
    }
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

// ------------------------------------------------------------------ v2: pre-split operand images
// The rank-K update's operands are thin panels (L21: rows x K, U12: K x cols, K <= 128) that
// every output tile re-reads.  tc_split writes them once per update as hi/lo TF32 images laid
// out exactly like a shared-memory stage (K-major core matrices), so lud_tc_update2 moves each
// chunk with four cp.async.bulk copies (one elected producer thread, mbarrier complete_tx)
// instead of all threads loading, splitting and storing between MMA chunks.
//   image element (row rho of the panel, k index kap):
//     chunk c = kap / KC, part p (0 hi, 1 lo), group g = rho / 8, kq = (kap % KC) / 4,
//     float offset ((c * 2 + p) * NG + g) * (KC * 8) + kq * 32 + (rho % 8) * 4 + kap % 4
// so the 16 groups of a 128-row tile form one contiguous 16 * KC * 32-byte block per (c, p).
constexpr int KC2 = 16;   // K chunk of the v2 pipeline (8 KB per operand part)
constexpr int NS2 = 3;    // pipeline stages: 3 x 32 KB -> 2 CTAs per SM

// blockIdx.y = 0: A operand, rows [base, n) of columns [k0, k0+kk);  1: B operand, columns
// [base, n) of rows [k0, k0+kk) (stored transposed: B^T K-major).  Entries outside the matrix
// or beyond kk are zero; ng = number of 8-row groups in the image.
__global__ void __launch_bounds__(256) tc_split(float* const* __restrict__ slot, int n, float* __restrict__ img_a,
                                                float* __restrict__ img_b, int base, int k0, int kk, int ng,
                                                int nchunks) {
    const float* A = *slot;
    const int which = blockIdx.y;  // 0: A image, 1: B image (one launch builds both)
    float* __restrict__ img = which == 0 ? img_a : img_b;
    const int kq_per = nchunks * (KC2 / 4);
    const int total = ng * 8 * kq_per;
    for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < total; e += gridDim.x * blockDim.x) {
        int rho, kqa;
        if (which == 0) { rho = e / kq_per; kqa = e - rho * kq_per; }       // k fastest: row reads
        else { kqa = e / (ng * 8); rho = e - kqa * (ng * 8); }              // column fastest
        const int idx = base + rho, kap = 4 * kqa;
        float v[4] = {0.f, 0.f, 0.f, 0.f};
        if (idx < n) {
#pragma unroll
            for (int q = 0; q < 4; ++q)
                if (kap + q < kk)
                    v[q] = which == 0 ? A[(size_t)idx * n + k0 + kap + q] : A[(size_t)(k0 + kap + q) * n + idx];
        }
        float4 h, l;
        split_tf32(v[0], h.x, l.x); split_tf32(v[1], h.y, l.y);
        split_tf32(v[2], h.z, l.z); split_tf32(v[3], h.w, l.w);
        const int c = kap / KC2, kq = (kap % KC2) / 4, g = rho >> 3, rr = rho & 7;
        const size_t off_hi = ((size_t)(c * 2) * ng + g) * (KC2 * 8) + kq * 32 + rr * 4;
        const size_t off_lo = ((size_t)(c * 2 + 1) * ng + g) * (KC2 * 8) + kq * 32 + rr * 4;
        *reinterpret_cast<float4*>(img + off_hi) = h;
        *reinterpret_cast<float4*>(img + off_lo) = l;
    }
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(b))
                 : "memory");
}

struct Img {
    const float* a;   // A image (rows from a_base)
    const float* b;   // B image (columns from b_base)
    int a_base, b_base, nga, ngb;
    int c0;           // first K chunk of the image this update reads (chunks c0 .. c0+nchunks-1)
};

// Store 4 consecutive k values (kap % 4 == 0) of image row rho as hi/lo TF32 parts (the layout
// above); used by tc_split and by the panel kernel that writes the images as it solves.
__device__ __forceinline__ void img_store4(float* __restrict__ img, int ng, int rho, int kap, const float (&v)[4]) {
    float4 h, l;
    split_tf32(v[0], h.x, l.x); split_tf32(v[1], h.y, l.y);
    split_tf32(v[2], h.z, l.z); split_tf32(v[3], h.w, l.w);
    const int c = kap / KC2, kq = (kap % KC2) / 4, g = rho >> 3, rr = rho & 7;
    *reinterpret_cast<float4*>(img + ((size_t)(c * 2) * ng + g) * (KC2 * 8) + kq * 32 + rr * 4) = h;
    *reinterpret_cast<float4*>(img + ((size_t)(c * 2 + 1) * ng + g) * (KC2 * 8) + kq * 32 + rr * 4) = l;
}

// C -= A*B on 128 x 128 tiles: warp 0 lane 0 produces (bulk copies into an NS2-stage ring),
// warp 1 lane 0 issues the 3xTF32 MMAs into TMEM and releases stages with tcgen05.commit; all
// four warps run the epilogue (tcgen05.ld, C -= acc in place).
__global__ void __launch_bounds__(128) lud_tc_update2(float* const* __restrict__ slot, int n, Args args, Img im) {
    constexpr int PART = BM * KC2 * 4;
    constexpr int STAGE = 4 * PART;
    constexpr uint32_t SBO = KC2 * 32;
    extern __shared__ __align__(1024) uint8_t sm[];
    uint64_t* full = reinterpret_cast<uint64_t*>(sm + NS2 * STAGE);
    uint64_t* empty = full + NS2;
    uint64_t* done = empty + NS2;
    uint32_t* tslot = reinterpret_cast<uint32_t*>(done + 1);
    float* A = *slot;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;

    int b = blockIdx.x, ri = 0;
    if (args.nrect == 2 && b >= args.rect[0].tiles) { b -= args.rect[0].tiles; ri = 1; }
    const Rect rc = ri ? args.rect[1] : args.rect[0];
    const int ty = b / rc.tiles_x, tx = b - ty * rc.tiles_x;
    const int row0 = rc.r0 + ty * BM, col0 = rc.c0 + tx * BN;
    const int rend = rc.r0 + rc.m, cend = rc.c0 + rc.nn;
    const bool vec = (n & 3) == 0;
    const int nchunks = (rc.kk + KC2 - 1) / KC2;
    const int ga = (row0 - im.a_base) >> 3, gb = (col0 - im.b_base) >> 3;

    if (tid == 0) {
        for (int i = 0; i < NS2; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
        mbar_init(done, 1);
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

    if (tid == 0) {  // producer
        for (int c = 0; c < nchunks; ++c) {
            const int s = c % NS2;
            if (c >= NS2) mbar_wait(&empty[s], ((c / NS2) - 1) & 1);
            uint8_t* st = sm + s * STAGE;
            mbar_expect_tx(&full[s], STAGE);
            const int ci = c + im.c0;
            const float* ah = im.a + ((size_t)(ci * 2) * im.nga + ga) * (KC2 * 8);
            const float* al = im.a + ((size_t)(ci * 2 + 1) * im.nga + ga) * (KC2 * 8);
            const float* bh = im.b + ((size_t)(ci * 2) * im.ngb + gb) * (KC2 * 8);
            const float* bl = im.b + ((size_t)(ci * 2 + 1) * im.ngb + gb) * (KC2 * 8);
            bulk_g2s(st, ah, PART, &full[s]);
            bulk_g2s(st + PART, al, PART, &full[s]);
            bulk_g2s(st + 2 * PART, bh, PART, &full[s]);
            bulk_g2s(st + 3 * PART, bl, PART, &full[s]);
        }
    } else if (tid == 32) {  // MMA issuer
        for (int c = 0; c < nchunks; ++c) {
            const int s = c % NS2;
            mbar_wait(&full[s], (c / NS2) & 1);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            const uint32_t a_hi = smem_u32(sm + s * STAGE), a_lo = a_hi + PART, b_hi = a_hi + 2 * PART,
                           b_lo = a_hi + 3 * PART;
#pragma unroll
            for (int ks = 0; ks < KC2 / 8; ++ks) {
                const uint64_t adh = sm_desc(a_hi + ks * 256, 128, SBO), adl = sm_desc(a_lo + ks * 256, 128, SBO);
                const uint64_t bdh = sm_desc(b_hi + ks * 256, 128, SBO), bdl = sm_desc(b_lo + ks * 256, 128, SBO);
                mma_tf32(tmem, adl, bdh, (c | ks) != 0);
                mma_tf32(tmem, adh, bdl, 1);
                mma_tf32(tmem, adh, bdh, 1);
            }
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                             smem_u32(&empty[s]))
                         : "memory");
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                         smem_u32(done))
                     : "memory");
    }
    __syncwarp();
    mbar_wait(done, 0);
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");

    const int r = row0 + warp * 32 + lane;
    const int ncols = min(BN, cend - col0);
    if (vec && (ncols & 3) == 0) {
        // Epilogue through the L2: -acc rows staged in the (now idle) pipeline shared memory,
        // then one bulk reduce-add (cp.reduce.async.bulk .add.f32) per row into C.  x + (-y) is
        // x - y bit for bit, each element is added exactly once, and the SMs never read C.
        constexpr int PITCH = BN * 4 + 16;  // 528 B: conflict-free 16-byte row-per-lane stores
        uint8_t* row_s = sm + (warp * 32 + lane) * PITCH;
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
            asm volatile("tcgen05.wait::ld.sync.aligned;"
                         : "+r"(v[0]), "+r"(v[1]), "+r"(v[2]), "+r"(v[3]), "+r"(v[4]), "+r"(v[5]), "+r"(v[6]),
                           "+r"(v[7]), "+r"(v[8]), "+r"(v[9]), "+r"(v[10]), "+r"(v[11]), "+r"(v[12]), "+r"(v[13]),
                           "+r"(v[14]), "+r"(v[15]), "+r"(v[16]), "+r"(v[17]), "+r"(v[18]), "+r"(v[19]),
                           "+r"(v[20]), "+r"(v[21]), "+r"(v[22]), "+r"(v[23]), "+r"(v[24]), "+r"(v[25]),
                           "+r"(v[26]), "+r"(v[27]), "+r"(v[28]), "+r"(v[29]), "+r"(v[30]), "+r"(v[31])
                         :
                         : "memory");
#pragma unroll
            for (int q = 0; q < 8; ++q)
                *reinterpret_cast<float4*>(row_s + jb * 128 + q * 16) =
                    make_float4(-__uint_as_float(v[4 * q]), -__uint_as_float(v[4 * q + 1]),
                                -__uint_as_float(v[4 * q + 2]), -__uint_as_float(v[4 * q + 3]));
        }
        // generic-proxy writes -> async proxy (bulk copy engine) reads
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        if (r < rend)
            asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f32 [%0], [%1], %2;" ::"l"(
                             A + (size_t)r * n + col0),
                         "r"(smem_u32(row_s)), "r"(ncols * 4)
                         : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    } else
    for (int jb = 0; jb < BN / 32; ++jb) {  // ragged or unaligned C: RMW per row
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

constexpr size_t smem_bytes2() { return (size_t)NS2 * 4 * BM * KC2 * 4 + 128; }

// v3 (round 2): the update with a BNT-wide C tile (128 or 256 columns; M = 128, accumulator
// 128 lanes x BNT TMEM columns).  A 128 x 256 tile reads the same A panel once for twice the
// outputs (the per-tile re-reads of the hi/lo panels from L2 are what bounded the 128 x 128
// version on large trailing matrices); stages hold A hi/lo + B hi/lo of one 16-deep K chunk
// (3 stages at 128 columns, 2 at 256: 96 KB, 2 CTAs and 2 x BNT <= 512 TMEM columns per SM).
template <int BNT>
struct Upd3 {
    static constexpr int NS = BNT == 256 ? 2 : 3;
    static constexpr int PA = BM * KC2 * 4;
    static constexpr int PB = BNT * KC2 * 4;
    static constexpr int STAGE = 2 * PA + 2 * PB;
    static constexpr size_t smem() { return (size_t)NS * STAGE + 128; }
    // kind::tf32, D f32, A and B K-major, M = 128, N = BNT
    static constexpr uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(BNT >> 3) << 17) |
                                      ((uint32_t)(BM >> 4) << 24);
};
__device__ __forceinline__ void mma_tf32_i(uint32_t tmem, uint64_t ad, uint64_t bd, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(tmem),
        "l"(ad), "l"(bd), "r"(idesc), "r"(acc));
}

template <int BNT>
__global__ void __launch_bounds__(128) lud_tc_update3(float* const* __restrict__ slot, int n, Args args, Img im) {
    constexpr int NS = Upd3<BNT>::NS;
    constexpr int PART = Upd3<BNT>::PA;   // one A part (hi or lo): 128 rows x KC2
    constexpr int PARTB = Upd3<BNT>::PB;  // one B part: BNT columns x KC2
    constexpr int STAGE = Upd3<BNT>::STAGE;
    constexpr uint32_t SBO = KC2 * 32;
    extern __shared__ __align__(1024) uint8_t sm[];
    uint64_t* full = reinterpret_cast<uint64_t*>(sm + NS * STAGE);
    uint64_t* empty = full + NS;
    uint64_t* done = empty + NS;
    uint32_t* tslot = reinterpret_cast<uint32_t*>(done + 1);
    asm volatile("griddepcontrol.wait;" ::: "memory");  // (a programmatic dependent on the chain)
    float* A = *slot;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;

    int b = blockIdx.x, ri = 0;
    if (args.nrect == 2 && b >= args.rect[0].tiles) { b -= args.rect[0].tiles; ri = 1; }
    const Rect rc = ri ? args.rect[1] : args.rect[0];
    const int ty = b / rc.tiles_x, tx = b - ty * rc.tiles_x;
    const int row0 = rc.r0 + ty * BM, col0 = rc.c0 + tx * BNT;
    const int rend = rc.r0 + rc.m, cend = rc.c0 + rc.nn;
    const bool vec = (n & 3) == 0;
    const int nchunks = (rc.kk + KC2 - 1) / KC2;
    const int ga = (row0 - im.a_base) >> 3, gb = (col0 - im.b_base) >> 3;

    if (tid == 0) {
        for (int i = 0; i < NS; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
        mbar_init(done, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tslot)), "n"(BNT));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = *tslot;

    if (tid == 0) {  // producer
        for (int c = 0; c < nchunks; ++c) {
            const int s = c % NS;
            if (c >= NS) mbar_wait(&empty[s], ((c / NS) - 1) & 1);
            uint8_t* st = sm + s * STAGE;
            mbar_expect_tx(&full[s], STAGE);
            const int ci = c + im.c0;
            const float* ah = im.a + ((size_t)(ci * 2) * im.nga + ga) * (KC2 * 8);
            const float* al = im.a + ((size_t)(ci * 2 + 1) * im.nga + ga) * (KC2 * 8);
            const float* bh = im.b + ((size_t)(ci * 2) * im.ngb + gb) * (KC2 * 8);
            const float* bl = im.b + ((size_t)(ci * 2 + 1) * im.ngb + gb) * (KC2 * 8);
            bulk_g2s(st, ah, PART, &full[s]);
            bulk_g2s(st + PART, al, PART, &full[s]);
            bulk_g2s(st + 2 * PART, bh, PARTB, &full[s]);
            bulk_g2s(st + 2 * PART + PARTB, bl, PARTB, &full[s]);
        }
    } else if (tid == 32) {  // MMA issuer
        for (int c = 0; c < nchunks; ++c) {
            const int s = c % NS;
            mbar_wait(&full[s], (c / NS) & 1);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            const uint32_t a_hi = smem_u32(sm + s * STAGE), a_lo = a_hi + PART, b_hi = a_hi + 2 * PART,
                           b_lo = b_hi + PARTB;
#pragma unroll
            for (int ks = 0; ks < KC2 / 8; ++ks) {
                const uint64_t adh = sm_desc(a_hi + ks * 256, 128, SBO), adl = sm_desc(a_lo + ks * 256, 128, SBO);
                const uint64_t bdh = sm_desc(b_hi + ks * 256, 128, SBO), bdl = sm_desc(b_lo + ks * 256, 128, SBO);
                mma_tf32_i(tmem, adl, bdh, Upd3<BNT>::idesc, (c | ks) != 0);
                mma_tf32_i(tmem, adh, bdl, Upd3<BNT>::idesc, 1);
                mma_tf32_i(tmem, adh, bdh, Upd3<BNT>::idesc, 1);
            }
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                             smem_u32(&empty[s]))
                         : "memory");
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                         smem_u32(done))
                     : "memory");
    }
    __syncwarp();
    mbar_wait(done, 0);
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");  // the next kernel may launch (it waits)

    const int r = row0 + warp * 32 + lane;
    const int ncols = min(BNT, cend - col0);
    if (vec && (ncols & 3) == 0) {
        // Epilogue through the L2, 128 columns at a time: -acc rows staged in the (now idle)
        // pipeline shared memory, then one bulk reduce-add (cp.reduce.async.bulk .add.f32) per
        // row into C.  x + (-y) is x - y bit for bit, each element is added exactly once, and
        // the SMs never read C.
        constexpr int PITCH = 128 * 4 + 16;  // 528 B: conflict-free 16-byte row-per-lane stores
        uint8_t* row_s = sm + (warp * 32 + lane) * PITCH;
#pragma unroll 1
        constexpr int HALF = BNT < 128 ? BNT : 128;  // columns staged per pass
        // C is read-modified-written once per update: mark it first to go from L2, so the
        // concurrently running chain kernels keep their code and operands there (their cold
        // instruction fetches otherwise come from HBM behind this stream)
        uint64_t c_policy;
        asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(c_policy));
        for (int h = 0; h < BNT / HALF; ++h) {
            const int nh = min(HALF, ncols - HALF * h);
            if (nh <= 0) break;  // CTA-uniform
            if (h > 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // row_s is free again
#pragma unroll 1
            for (int jb = 0; jb < HALF / 32; ++jb) {
                uint32_t v[32];
                const uint32_t taddr = tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)(HALF * h + jb * 32);
                asm volatile(
                    "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
                    "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                    : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
                      "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]),
                      "=r"(v[15]), "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]),
                      "=r"(v[22]), "=r"(v[23]), "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]),
                      "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
                    : "r"(taddr));
                asm volatile("tcgen05.wait::ld.sync.aligned;"
                             : "+r"(v[0]), "+r"(v[1]), "+r"(v[2]), "+r"(v[3]), "+r"(v[4]), "+r"(v[5]), "+r"(v[6]),
                               "+r"(v[7]), "+r"(v[8]), "+r"(v[9]), "+r"(v[10]), "+r"(v[11]), "+r"(v[12]), "+r"(v[13]),
                               "+r"(v[14]), "+r"(v[15]), "+r"(v[16]), "+r"(v[17]), "+r"(v[18]), "+r"(v[19]),
                               "+r"(v[20]), "+r"(v[21]), "+r"(v[22]), "+r"(v[23]), "+r"(v[24]), "+r"(v[25]),
                               "+r"(v[26]), "+r"(v[27]), "+r"(v[28]), "+r"(v[29]), "+r"(v[30]), "+r"(v[31])
                             :
                             : "memory");
#pragma unroll
                for (int q = 0; q < 8; ++q)
                    *reinterpret_cast<float4*>(row_s + jb * 128 + q * 16) =
                        make_float4(-__uint_as_float(v[4 * q]), -__uint_as_float(v[4 * q + 1]),
                                    -__uint_as_float(v[4 * q + 2]), -__uint_as_float(v[4 * q + 3]));
            }
            // generic-proxy writes -> async proxy (bulk copy engine) reads
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            if (r < rend)
                asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.L2::cache_hint.add.f32 [%0], [%1], %2, %3;"
                             ::"l"(A + (size_t)r * n + col0 + HALF * h),
                             "r"(smem_u32(row_s)), "r"(nh * 4), "l"(c_policy)
                             : "memory");
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        }
        asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    } else
    for (int jb = 0; jb < BNT / 32; ++jb) {  // ragged or unaligned C: RMW per row
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
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(BNT));
}



// v1 (single-thread-group staging, kept as the reference the layout probe
// tools/ubench/tc_dump.cu exercises; the library runs lud_tc_update2 above).
#ifndef RG_LUD_KC
#define RG_LUD_KC 16
#endif
constexpr int KC_MAIN = RG_LUD_KC;  // K chunk per stage: 16 -> 64 KB smem, 3 CTAs per SM
constexpr size_t smem_bytes(int kc) { return (size_t)2 * 4 * BM * kc * 4 + 64; }

inline Rect make_rect(int r0, int c0, int m, int nn, int k0, int kk, int bn = BN) {
    Rect r;
    r.r0 = r0; r.c0 = c0; r.m = m; r.nn = nn; r.k0 = k0; r.kk = kk;
    r.tiles_x = (nn + bn - 1) / bn;
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

// Scratch for the v2 operand images: (n + 256) rows x 128 k x hi/lo floats each.
inline size_t img_floats(int n) { return (size_t)(n + 256) * 128 * 2; }

// v2: split the panels of rows/cols [base, n) x k [k0, k0+kk) into the images, then C -= A*B
// over the rectangles (whose row and column starts are base + multiples of 8).
inline void launch_update2(float* const* slot, int n, const Rect* rs, int nr, int base, float* img_a, float* img_b,
                           cudaStream_t s) {
    Args a;
    a.nrect = 0;
    for (int i = 0; i < nr; ++i)
        if (rs[i].m > 0 && rs[i].nn > 0 && rs[i].kk > 0) a.rect[a.nrect++] = rs[i];
    if (a.nrect == 0) return;
    if (a.nrect == 1) a.rect[1] = a.rect[0];
    const int k0 = a.rect[0].k0, kk = a.rect[0].kk;
    const int nchunks = (kk + KC2 - 1) / KC2;
    const int ng = ((n - base + 127) / 128 + 1) * 16;  // padded to whole tiles + one spare tile
    const int total = ng * 8 * nchunks * (KC2 / 4);
    const int grid_s = std::min((total + 255) / 256, 148 * 8);
    tc_split<<<dim3(grid_s, 2), 256, 0, s>>>(slot, n, img_a, img_b, base, k0, kk, ng, nchunks);
    Img im{img_a, img_b, base, base, ng, ng, 0};
    const int grid = a.rect[0].tiles + (a.nrect == 2 ? a.rect[1].tiles : 0);
    lud_tc_update2<<<grid, 128, smem_bytes2(), s>>>(slot, n, a, im);
}

}  // namespace tc
}  // namespace rg

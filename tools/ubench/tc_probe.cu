// Probes for the tcgen05 path (development aid): (1) TMEM st/ld round trip, (2) one MMA on
// all-ones operands in the canonical no-swizzle layouts (expect acc = 8 everywhere).
#include <cstdio>
#include "lud_tc.cuh"
using namespace rg;
using namespace rg::tc;
__global__ void probe(float* out, int mode) {
    __shared__ __align__(1024) uint8_t sm[4 * 128 * 8 * 4 + 64];  // 16 KB operands
    __shared__ uint64_t mbar;
    __shared__ uint32_t tslot;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    if (tid == 0) { mbar_init(&mbar, 1); asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" ::"r"(smem_u32(&tslot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = tslot;
    if (mode == 0) {
        uint32_t v = __float_as_uint((float)(warp * 32 + lane) * 1000.f + 7.f);
        asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(tmem + ((uint32_t)(warp * 32) << 16) + 7), "r"(v));
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    } else {
        {   // sentinel 5.0 in every column this warp's lanes own
            const uint32_t five = __float_as_uint(5.0f);
            for (int c = 0; c < 32; ++c)
                asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(tmem + ((uint32_t)(warp * 32) << 16) + c), "r"(five));
            asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        }
        // A part (128 x 8, K-major) and B part (8 x 128, MN-major) = 4 KB each; fill with 1.0
        float* f = reinterpret_cast<float*>(sm);
        if (mode == 3) {  // bf16 ones, kind::f16 (K = 16 per instruction, same byte geometry)
            uint32_t* u = reinterpret_cast<uint32_t*>(sm);
            for (int e = tid; e < 2 * 128 * 8; e += 128) u[e] = 0x3F803F80u;
        } else if (mode >= 4) {
            for (int e = tid; e < 4 * 128 * 8; e += 128) f[e] = 1.0f;
        } else
            for (int e = tid; e < 2 * 128 * 8; e += 128) f[e] = (mode == 2 && e >= 1024) ? (float)((e - 1024) / 32) : 1.0f;
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncthreads();
        if (tid == 0) {
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            const uint32_t a = smem_u32(sm), b = a + 4096;
            if (mode == 3) {
                const uint32_t idf16 = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 16) | (16u << 17) | (8u << 24);
                asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                             "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(tmem),
                             "l"(sm_desc(a, 128, 256)), "l"(sm_desc(b, 128, 128)), "r"(idf16), "r"(0));
            } else if (mode >= 4) {
                uint32_t id = (1u << 4) | (2u << 7) | (2u << 10) | (16u << 17) | (8u << 24);  // both K-major
                if (mode == 5) id |= 1u << 16;
                if (mode == 6) id = (1u << 4) | (0u << 7) | (0u << 10) | (16u << 17) | (8u << 24);
                if (mode == 7) id = (1u << 4) | (2u << 7) | (2u << 10) | (16u << 17) | (4u << 24);
                asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                             "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(tmem),
                             "l"(sm_desc(a, 128, 256)), "l"(sm_desc(b, 128, 256)), "r"(id), "r"(0));
            } else
                mma_tf32(tmem, sm_desc(a, 128, 256), sm_desc(b, 128, 128), 0);
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&mbar)) : "memory");
        }
        mbar_wait(&mbar, 0);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    }
    uint32_t v[32];
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]),
          "=r"(v[15]), "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]),
          "=r"(v[22]), "=r"(v[23]), "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]),
          "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
        : "r"(tmem + ((uint32_t)(warp * 32) << 16)));
    asm volatile("tcgen05.wait::ld.sync.aligned;" : "+r"(v[0]), "+r"(v[7]), "+r"(v[1]), "+r"(v[31]) :: "memory");
    for (int j = 0; j < 32; ++j) out[(warp * 32 + lane) * 32 + j] = __uint_as_float(v[j]);
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" ::"r"(tmem));
}
int main() {
    float* d; cudaMalloc(&d, 128 * 32 * 4);
    float h[128 * 32];
    for (int mode = 0; mode < 8; ++mode) {
        cudaMemset(d, 0, 128 * 32 * 4);
        probe<<<1, 128>>>(d, mode);
        cudaError_t e = cudaDeviceSynchronize();
        cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
        printf("tmem probe ");
        printf("mode %d (%s): row0 %g %g %g %g ... [0][7]=%g  row1[7]=%g row64[7]=%g row127: %g %g %g\n", mode, cudaGetErrorString(e),
               h[0], h[1], h[2], h[3], h[7], h[32 + 7], h[64 * 32 + 7], h[127 * 32], h[127 * 32 + 1], h[127 * 32 + 31]);
    }
    return 0;
}

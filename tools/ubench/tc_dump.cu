// Layout check for the tcgen05 rank-K update (lud_tc.cuh): runs C -= A*B on a 256 x 256 matrix
// (A = rows 128.., cols 0..kk; B = rows 0..kk, cols 128..; C = rows/cols 128..) for several kk
// and dumps before/after as raw fp32 for offline comparison.  Development aid.
#include <cstdio>
#include <cstdlib>
#include <vector>
#include "lud_tc.cuh"
using namespace rg;
int main(int argc, char** argv) {
    const char* out = argc > 1 ? argv[1] : "tc_dump";
    const int n = 256;
    std::vector<float> h(n * n);
    srand(1);
    for (auto& x : h) x = (float)(rand() % 2001 - 1000) / 256.0f;  // exact in TF32? no: 11 bits
    float *d, **slot;
    cudaMalloc(&d, n * n * 4);
    cudaMalloc(&slot, sizeof(float*));
    cudaMemcpy(slot, &d, sizeof(float*), cudaMemcpyHostToDevice);
    cudaFuncSetAttribute(tc::lud_tc_update<tc::KC_MAIN>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)tc::smem_bytes(tc::KC_MAIN));
    char fn[256];
    snprintf(fn, sizeof fn, "%s_in.bin", out);
    FILE* f = fopen(fn, "wb"); fwrite(h.data(), 4, n * n, f); fclose(f);
    for (int kk : {8, 16, 32, 100}) {
        cudaMemcpy(d, h.data(), n * n * 4, cudaMemcpyHostToDevice);
        tc::Rect r = tc::make_rect(128, 128, 128, 128, 0, kk);
        tc::launch_update(slot, n, &r, 1, 0);
        cudaError_t e = cudaDeviceSynchronize();
        printf("kk=%d: %s\n", kk, cudaGetErrorString(e));
        std::vector<float> o(n * n);
        cudaMemcpy(o.data(), d, n * n * 4, cudaMemcpyDeviceToHost);
        snprintf(fn, sizeof fn, "%s_k%d.bin", out, kk);
        f = fopen(fn, "wb"); fwrite(o.data(), 4, n * n, f); fclose(f);
    }
    return 0;
}

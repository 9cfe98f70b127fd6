// workloads.h -- internal interfaces shared between the workload TUs and the multi-GPU
// row-slab layer (dist.cu).  Not part of the C ABI.
#pragma once

#include <cuda_runtime.h>

#include "hs_cell.cuh"
#include "rg_internal.h"

namespace rg {

// ------------------------------------------------------------------ hotspot (hotspot.cu)
namespace hotspot {
struct DirectVariant;
struct StreamVariant;
rodinia_status check(const rodinia_granularity& g, int64_t R, int64_t C, const DirectVariant** dv,
                     const StreamVariant** sv);
// Steps in state space (u = T - amb, kP = k*P; hs_cell.cuh): usrc -> udst via uscr.
rodinia_status run(const float* usrc, const float* kp, float* udst, float* uscr, int R, int C, int iters,
                   const HsCoef& cf, const rodinia_granularity& g, const DirectVariant* dv,
                   const StreamVariant* sv, cudaStream_t s);
// Whole solve from temperatures (conversions + run); scr and kp are R x C scratch buffers.
rodinia_status solve(const float* tin, const float* p, float* tout, float* scr, float* kp, int R, int C,
                     int iters, const rodinia_hotspot_coeffs& cc, const rodinia_granularity& g,
                     const DirectVariant* dv, const StreamVariant* sv, cudaStream_t s);
// Elementwise state conversions: op 0: y = x - a, 1: y = x * a, 2: y = x + a (in place allowed).
void convert(const float* x, float* y, int64_t n, int op, float a, cudaStream_t s);
int num_launches(int iters, const StreamVariant* sv);
int temporal_of(const StreamVariant* sv);  // steps per launch (1 for the direct family)
}  // namespace hotspot

// ------------------------------------------------------------------ srad (srad.cu)
struct SradIter {       // written by srad_roi_stats, read by the pass kernels
    float q0;           // q0sqr rounded to fp32
    float r0;           // 1 / (q0 * (1 + q0))
    int degenerate;     // ROI mean == 0
    int pad;
};

namespace srad {
typedef void (*FusedFn)(const float*, float*, int, int, int, int, float, const SradIter*);
struct Variant { int tx, ty, mode; FusedFn fn; const char* key; };
typedef void (*StreamFn)(const float*, float*, int, int, int, int, float, const SradIter*, int);
struct StreamVariant { int v, occ; StreamFn fn; const char* key; };
// Plan: dataflow (uncoarsened) iff granularity is exactly the uncoarsened one.
struct Plan {
    bool dataflow;
    const Variant* v;
    const StreamVariant* stream;   // stream family (flags & RODINIA_STREAM)
    int bx, by;
    size_t smem;
};

struct Engine {  // library-owned scratch for one solve
    Plan p;
    int R = 0, C = 0;
    SradIter* its = nullptr;                // per-iteration q0sqr / reciprocal / degenerate flag
    double2* partials = nullptr;
    unsigned* counter = nullptr;
    int* sticky = nullptr;
    float* jb = nullptr;                    // ping-pong partner of J
    float* df[5] = {nullptr, nullptr, nullptr, nullptr, nullptr};  // dataflow arrays
    char* blob = nullptr;
};

rodinia_status plan(const rodinia_granularity& g, Plan* p);
rodinia_status engine_alloc(Engine* e, const Plan& p, int R, int C, int niter, cudaStream_t s);
void engine_free(Engine* e, cudaStream_t s);
float* engine_steps(Engine* e, float* cur, float* other, int i0, int i1, bool stats, int r1, int c1,
                    int rw, int cw, float lam4, cudaStream_t s);
rodinia_status take_sticky();
}  // namespace srad

// 2-D block-cyclic distributed LU building blocks (lud.cu; orchestrated by rodinia_lud_dist)
namespace ldist {
constexpr int NB = 128;                      // block size (the tensor-core update tile)
size_t mimg_floats();                        // diagonal-block payload (U, L^T images, 1/u)
int img_groups(int64_t rows);                // 8-row groups of an operand image for `rows`
size_t img_floats(int64_t rows);             // floats of such an image (hi + lo, K = 128)
// The matrix pointer is read on the device from *slot (CUDA-graph reuse); off = element offset.
// prio: cudaLaunchAttributePriority of the launch (0 = none; graph capture keeps it per node)
rodinia_status diag(float* const* slot, size_t off, int lda, int r, float* mimg, cudaStream_t s, int prio = 0);
struct TrsmJob {        // L rows (lower = 1: row t at A + t*lda) or U columns (column t at A + t),
    float* const* slot;    // A = *slot + off
    size_t off;
    int lda, lower, count;
    float* img;            // operand image (ng 8-row groups), image row = thread index
    int ng;
};
rodinia_status trsm(const TrsmJob* job, int njobs, const float* mimg, cudaStream_t s, int prio = 0);  // one launch
rodinia_status set_slot(float** slot, float* a, cudaStream_t s);
// A -= L U over up to two rectangles rect[i] = {r0, m, c0, nn} of the local matrix; the operand
// images start at local row a_base / column b_base (the trailing part's first row / column)
rodinia_status update(float* const* slot, int lda, const int (*rect)[4], int nr, int a_base, const float* ia,
                      int nga, int b_base, const float* ib, int ngb, cudaStream_t s, int prio = 0, int kk = NB,
                      int c0 = 0);  // kk: update rank (128, or 256 over two steps' images); c0: first image chunk
}  // namespace ldist

}  // namespace rg

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
rodinia_status run(const float* tin, const float* p, float* tout, float* scr, int R, int C, int iters,
                   const HsCoef& cf, const rodinia_granularity& g, const DirectVariant* dv,
                   const StreamVariant* sv, cudaStream_t s);
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
struct StreamVariant { int v; StreamFn fn; const char* key; };
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

}  // namespace rg

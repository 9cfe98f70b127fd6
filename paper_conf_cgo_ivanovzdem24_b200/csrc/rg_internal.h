// rg_internal.h -- internal helpers of librodinia_gran.so (not part of the C ABI).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <mutex>
#include <string>
#include <vector>

#include "rodinia_gran.h"

namespace rg {

// ------------------------------------------------------------------ errors
rodinia_status set_error(rodinia_status s, const char* fmt, ...);
rodinia_status cuda_error(cudaError_t e, const char* what, const char* file, int line);
void clear_error();

#define RG_CUDA(x)                                                                      \
    do {                                                                                \
        cudaError_t _rg_e = (x);                                                        \
        if (_rg_e != cudaSuccess) return ::rg::cuda_error(_rg_e, #x, __FILE__, __LINE__); \
    } while (0)

#define RG_TRY(x)                                \
    do {                                         \
        rodinia_status _rg_s = (x);              \
        if (_rg_s != RODINIA_OK) return _rg_s;   \
    } while (0)

extern std::atomic<int64_t> g_launches;
inline void count_launch(int64_t n = 1) { g_launches.fetch_add(n, std::memory_order_relaxed); }
// Dominant-kernel timing (rodinia_kernel_timing): event pair around a stepping launch.
void ktime_begin(cudaStream_t s);
void ktime_end(cudaStream_t s);

// ------------------------------------------------------------------ device
struct DeviceInfo {
    int device = -1;
    int sms = 0;
    int smem_optin = 0;       // max dynamic+static smem per CTA (opt-in)
    int smem_per_sm = 0;
    int regs_per_sm = 0;
    int l2_bytes = 0;
    int cc_major = 0, cc_minor = 0;
    char name[256] = {0};
};
// Requires a device; returns RODINIA_E_NODEV when none.
rodinia_status device_info(DeviceInfo* out);

// ------------------------------------------------------------------ variants
// ptxas statistics of one kernel instantiation, generated at build time by
// tools/ptxas_filter.py into variant_stats.cpp (key = demangled name incl. template args).
struct PtxasStats {
    const char* key;
    int regs, spill_stores, spill_loads, stack, smem;
};
const PtxasStats* find_stats(const char* key);  // nullptr if unknown

// Compile-time filter decision: returns RODINIA_OK or the pruning status.
// `base_spill` is the spill bytes of the family's uncoarsened kernel (new spills are pruned).
rodinia_status filter_decision(const PtxasStats* st, int threads, int smem_bytes, int base_spill);

// The filter applied at the boundary to an explicitly requested instantiation: RODINIA_OK, or
// RODINIA_E_FILTERED / RODINIA_E_SMEM with a message, unless flags & RODINIA_FORCE.
rodinia_status boundary_filter(rodinia_kernel k, const char* key, int threads, int dyn_smem, int flags);

// Occupancy query (CTAs / SM) of a kernel at block size and dynamic smem; 0 on failure.
int ctas_per_sm(const void* func, int threads, size_t dyn_smem);

// ------------------------------------------------------------------ granularity helpers
inline bool gran_is_zero(const rodinia_granularity* g) {
    return !g || (g->thread_x == 0 && g->thread_y == 0 && g->block_x == 0 && g->block_y == 0 &&
                  g->temporal == 0 && g->index_mode == 0 && g->flags == 0);
}
inline rodinia_granularity gran(int tx, int ty, int bx, int by, int h, int mode, int flags = 0) {
    rodinia_granularity g;
    g.thread_x = tx; g.thread_y = ty; g.block_x = bx; g.block_y = by;
    g.temporal = h; g.index_mode = mode; g.flags = flags;
    return g;
}
std::string gran_str(const rodinia_granularity& g);

// Default granularity per workload when neither the caller nor the tune cache chooses one.
rodinia_granularity default_gran(rodinia_kernel k, const rodinia_problem& p);

// Cached device buffers of the *_host entry points (index 0..2), grown on demand.  The caller
// holds host_mutex() for the whole H2D / solve / D2H / sync sequence that uses them.
rodinia_status host_buffer(int i, size_t bytes, void** out);
std::mutex& host_mutex();

// ------------------------------------------------------------------ pre-pruning (tune.cu, model.cu)
// Model estimate of one call at row.g (rodinia_model_ms); -1 when the workload is not modelled.
float model_estimate_ms(rodinia_kernel k, const rodinia_problem& p, const rodinia_tune_row& row);
// Called by every tuner after the compile-time filter, before timing a candidate: fills
// row->model_ms and returns RODINIA_OK to time it or RODINIA_E_PRUNED (rodinia_tune_pruned).
rodinia_status prune_gate(rodinia_kernel k, const rodinia_problem& p, rodinia_tune_row* row);
bool prune_active();

// ------------------------------------------------------------------ tune cache
bool tune_cache_lookup(rodinia_kernel k, const rodinia_problem& p, rodinia_granularity* out);
void tune_cache_store(rodinia_kernel k, const rodinia_problem& p, const rodinia_granularity& g,
                      float ms);

// ------------------------------------------------------------------ scratch
// Stream-ordered scratch allocation (cudaMallocAsync from the device's default pool, whose
// release threshold is raised once so repeated calls reuse memory).
rodinia_status scratch_alloc(void** p, size_t bytes, cudaStream_t s);
void scratch_free(void* p, cudaStream_t s);

}  // namespace rg

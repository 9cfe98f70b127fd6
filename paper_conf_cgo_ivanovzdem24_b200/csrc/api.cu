// api.cu -- exported C ABI (include/rodinia_gran.h): errors, device info, scratch, filter,
// tune cache and the hotspot entry points.  Other workloads live in their own TUs.
#include <cuda_runtime.h>
#include <stdarg.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <cmath>
#include <fstream>
#include <mutex>
#include <sstream>
#include <string>
#include <vector>

#include "hs_cell.cuh"
#include "workloads.h"
#include "rg_internal.h"

namespace rg {

std::atomic<int64_t> g_launches{0};

static thread_local std::string t_last_error;

rodinia_status set_error(rodinia_status s, const char* fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    t_last_error = buf;
    return s;
}

void clear_error() { t_last_error.clear(); }

rodinia_status cuda_error(cudaError_t e, const char* what, const char* file, int line) {
    rodinia_status s = RODINIA_E_CUDA;
    if (e == cudaErrorNoDevice || e == cudaErrorInsufficientDriver) s = RODINIA_E_NODEV;
    if (e == cudaErrorMemoryAllocation) s = RODINIA_E_NOMEM;
    return set_error(s, "%s failed: %s (%s:%d)", what, cudaGetErrorString(e), file, line);
}

std::string gran_str(const rodinia_granularity& g) {
    char b[160];
    snprintf(b, sizeof b, "t=(%d,%d) b=(%d,%d) h=%d mode=%d flags=%d", g.thread_x, g.thread_y,
             g.block_x, g.block_y, g.temporal, g.index_mode, g.flags);
    return b;
}

// ------------------------------------------------------------------ device
rodinia_status device_info(DeviceInfo* out) {
    static std::mutex mu;
    static DeviceInfo cache[64];
    int dev = -1;
    int count = 0;
    cudaError_t e = cudaGetDeviceCount(&count);
    if (e != cudaSuccess || count == 0) {
        cudaGetLastError();
        return set_error(RODINIA_E_NODEV, "no CUDA device available (%s)",
                         e == cudaSuccess ? "0 devices" : cudaGetErrorString(e));
    }
    RG_CUDA(cudaGetDevice(&dev));
    std::lock_guard<std::mutex> lk(mu);
    DeviceInfo& d = cache[dev & 63];
    if (d.device != dev) {
        cudaDeviceProp prop;
        RG_CUDA(cudaGetDeviceProperties(&prop, dev));
        d.sms = prop.multiProcessorCount;
        d.smem_optin = (int)prop.sharedMemPerBlockOptin;
        d.smem_per_sm = (int)prop.sharedMemPerMultiprocessor;
        d.regs_per_sm = prop.regsPerMultiprocessor;
        d.l2_bytes = prop.l2CacheSize;
        d.cc_major = prop.major;
        d.cc_minor = prop.minor;
        snprintf(d.name, sizeof d.name, "%s", prop.name);
        // Stream-ordered scratch reuse: keep freed pool memory instead of returning it.
        cudaMemPool_t pool;
        if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
            uint64_t thr = UINT64_MAX;
            cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
        }
        cudaGetLastError();
        d.device = dev;
    }
    *out = d;
    return RODINIA_OK;
}

rodinia_status scratch_alloc(void** p, size_t bytes, cudaStream_t s) {
    DeviceInfo di;
    RG_TRY(device_info(&di));
    cudaError_t e = cudaMallocAsync(p, bytes, s);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return set_error(RODINIA_E_NOMEM, "cudaMallocAsync(%zu) failed: %s", bytes, cudaGetErrorString(e));
    }
    return RODINIA_OK;
}

void scratch_free(void* p, cudaStream_t s) {
    if (p) cudaFreeAsync(p, s);
}

int ctas_per_sm(const void* func, int threads, size_t dyn_smem) {
    int n = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, func, threads, dyn_smem) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    return n;
}

// ------------------------------------------------------------------ compile-time filter
rodinia_status filter_decision(const PtxasStats* st, int threads, int smem_bytes, int base_spill) {
    if (!st) return RODINIA_OK;  // unknown stats: not pruned (reported as regs = -1)
    const int spill = st->spill_stores + st->spill_loads;
    const int smem_limit = 227 * 1024;  // B200 opt-in max per CTA
    if (st->smem + smem_bytes > smem_limit) return RODINIA_E_SMEM;
    if (spill > 0 && base_spill == 0) return RODINIA_E_FILTERED;              // new spills
    if ((int64_t)st->regs * threads > 65536) return RODINIA_E_FILTERED;       // 0 CTAs / SM
    return RODINIA_OK;
}

// ------------------------------------------------------------------ tune cache
struct CacheEntry {
    std::string key;
    rodinia_granularity g;
};
static std::mutex g_cache_mu;
static std::vector<CacheEntry> g_cache;
static bool g_cache_loaded = false;

static std::string cache_key(rodinia_kernel k, const rodinia_problem& p) {
    DeviceInfo di;
    char b[512];
    const char* dev = "nodev";
    int sms = 0;
    if (device_info(&di) == RODINIA_OK) { dev = di.name; sms = di.sms; }
    snprintf(b, sizeof b, "%s|%d|%d|%lldx%lldx%d|%d|%d", dev, sms, (int)k, (long long)p.rows,
             (long long)p.cols, p.depth, p.iterations, p.nranks);
    return b;
}

static const char* cache_path() {
    const char* p = getenv("RODINIA_TUNE_CACHE");
    return (p && *p) ? p : nullptr;
}

static void cache_load_locked() {
    if (g_cache_loaded) return;
    g_cache_loaded = true;
    const char* path = cache_path();
    if (!path) return;
    std::ifstream f(path);
    std::string line;
    while (std::getline(f, line)) {
        // format: key \t tx ty bx by h mode flags \t ms
        size_t a = line.find('\t');
        if (a == std::string::npos) continue;
        CacheEntry e;
        e.key = line.substr(0, a);
        std::istringstream is(line.substr(a + 1));
        is >> e.g.thread_x >> e.g.thread_y >> e.g.block_x >> e.g.block_y >> e.g.temporal >>
            e.g.index_mode >> e.g.flags;
        if (!is) continue;
        bool replaced = false;
        for (auto& c : g_cache)
            if (c.key == e.key) { c = e; replaced = true; }
        if (!replaced) g_cache.push_back(e);
    }
}

bool tune_cache_lookup(rodinia_kernel k, const rodinia_problem& p, rodinia_granularity* out) {
    std::string key = cache_key(k, p);
    std::lock_guard<std::mutex> lk(g_cache_mu);
    cache_load_locked();
    for (auto& c : g_cache)
        if (c.key == key) { *out = c.g; return true; }
    return false;
}

void tune_cache_store(rodinia_kernel k, const rodinia_problem& p, const rodinia_granularity& g, float ms) {
    std::string key = cache_key(k, p);
    std::lock_guard<std::mutex> lk(g_cache_mu);
    cache_load_locked();
    bool replaced = false;
    for (auto& c : g_cache)
        if (c.key == key) { c.g = g; replaced = true; }
    if (!replaced) g_cache.push_back({key, g});
    const char* path = cache_path();
    if (!path) return;
    FILE* f = fopen(path, "a");
    if (!f) return;
    fprintf(f, "%s\t%d %d %d %d %d %d %d\t%.6f\n", key.c_str(), g.thread_x, g.thread_y, g.block_x,
            g.block_y, g.temporal, g.index_mode, g.flags, ms);
    fclose(f);
}

namespace hotspot {
struct DirectVariant;
struct StreamVariant;
}  // namespace hotspot

// Default granularity per workload when neither the caller nor the tune cache chooses one.
rodinia_granularity default_gran(rodinia_kernel k, const rodinia_problem& p);

}  // namespace rg

using namespace rg;

// ===================================================================== exported: misc
extern "C" const char* rodinia_last_error(void) { return t_last_error.c_str(); }

extern "C" const char* rodinia_status_string(rodinia_status s) {
    switch (s) {
        case RODINIA_OK: return "RODINIA_OK";
        case RODINIA_E_INVALID: return "RODINIA_E_INVALID";
        case RODINIA_E_ILLEGAL_FACTOR: return "RODINIA_E_ILLEGAL_FACTOR";
        case RODINIA_E_SMEM: return "RODINIA_E_SMEM";
        case RODINIA_E_FILTERED: return "RODINIA_E_FILTERED";
        case RODINIA_E_NOT_BUILT: return "RODINIA_E_NOT_BUILT";
        case RODINIA_E_DEGENERATE: return "RODINIA_E_DEGENERATE";
        case RODINIA_E_NODEV: return "RODINIA_E_NODEV";
        case RODINIA_E_CUDA: return "RODINIA_E_CUDA";
        case RODINIA_E_NCCL: return "RODINIA_E_NCCL";
        case RODINIA_E_NOMEM: return "RODINIA_E_NOMEM";
        case RODINIA_E_PRUNED: return "RODINIA_E_PRUNED";
    }
    return "RODINIA_E_UNKNOWN";
}

extern "C" int32_t rodinia_abi_version(void) { return RODINIA_ABI_VERSION; }
extern "C" int64_t rodinia_launch_count(void) { return g_launches.load(); }

// ---------------------------------------------------------------- dominant-kernel timing
namespace rg {
struct KTimer {
    std::mutex mu;
    bool on = false;
    std::vector<cudaEvent_t> pool;  // 2 per timed launch, reused across enables
    size_t used = 0;
};
static KTimer& ktimer() {
    static KTimer k;
    return k;
}
static cudaEvent_t ktime_event() {
    KTimer& k = ktimer();
    if (k.used == k.pool.size()) {
        cudaEvent_t e;
        if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
        k.pool.push_back(e);
    }
    return k.pool[k.used++];
}
void ktime_begin(cudaStream_t s) {
    KTimer& k = ktimer();
    std::lock_guard<std::mutex> lk(k.mu);
    if (!k.on) return;
    if (k.used % 2 == 1) return;  // unmatched begin: ignore
    cudaEvent_t e = ktime_event();
    if (e) cudaEventRecord(e, s);
}
void ktime_end(cudaStream_t s) {
    KTimer& k = ktimer();
    std::lock_guard<std::mutex> lk(k.mu);
    if (!k.on || k.used % 2 == 0) return;
    cudaEvent_t e = ktime_event();
    if (e) cudaEventRecord(e, s);
}
}  // namespace rg

extern "C" rodinia_status rodinia_kernel_timing(int32_t enable) {
    KTimer& k = ktimer();
    std::lock_guard<std::mutex> lk(k.mu);
    k.on = enable != 0;
    if (k.on) k.used = 0;
    return RODINIA_OK;
}

extern "C" rodinia_status rodinia_kernel_time(double* total_ms, int64_t* launches) {
    if (!total_ms || !launches) return set_error(RODINIA_E_INVALID, "kernel_time: null argument");
    KTimer& k = ktimer();
    std::lock_guard<std::mutex> lk(k.mu);
    double t = 0.0;
    const size_t n = k.used / 2;
    for (size_t i = 0; i < n; ++i) {
        RG_CUDA(cudaEventSynchronize(k.pool[2 * i + 1]));
        float ms = 0.f;
        RG_CUDA(cudaEventElapsedTime(&ms, k.pool[2 * i], k.pool[2 * i + 1]));
        t += ms;
    }
    *total_ms = t;
    *launches = (int64_t)n;
    return RODINIA_OK;
}

namespace rg { namespace srad { rodinia_status take_sticky(); } }

extern "C" rodinia_status rodinia_sync(void* stream) {
    DeviceInfo di;
    RG_TRY(device_info(&di));
    RG_CUDA(cudaStreamSynchronize((cudaStream_t)stream));
    RG_CUDA(cudaGetLastError());
    return srad::take_sticky();
}

// ===================================================================== exported: hotspot
extern "C" rodinia_status rodinia_hotspot_coeffs_rodinia(int64_t rows, int64_t cols, double chip_w,
                                                         double chip_h, rodinia_hotspot_coeffs* out) {
    if (rows < 1 || cols < 1 || !(chip_w > 0) || !(chip_h > 0) || !out || !std::isfinite(chip_w) ||
        !std::isfinite(chip_h))
        return set_error(RODINIA_E_INVALID, "hotspot_coeffs: bad arguments");
    // Rodinia hotspot constants (DESIGN.md §3 H1): t_chip, K_SI, SPEC_HEAT_SI, FACTOR_CHIP,
    // MAX_PD, PRECISION, amb.
    const double t_chip = 0.0005, k_si = 100.0, spec_heat = 1.75e6, factor_chip = 0.5;
    const double max_pd = 3.0e6, precision = 0.001;
    const double gw = chip_w / (double)cols, gh = chip_h / (double)rows;
    const double cap = factor_chip * spec_heat * t_chip * gw * gh;
    const double Rx = gw / (2.0 * k_si * t_chip * gh);
    const double Ry = gh / (2.0 * k_si * t_chip * gw);
    const double Rz = t_chip / (k_si * gh * gw);
    const double step = precision / (max_pd / (factor_chip * t_chip * spec_heat));
    out->k = (float)(step / cap);
    out->rx = (float)(1.0 / Rx);
    out->ry = (float)(1.0 / Ry);
    out->rz = (float)(1.0 / Rz);
    out->amb = 80.0f;
    return RODINIA_OK;
}

static rodinia_status hotspot_validate(const void* tin, const void* p, const void* tout, int64_t R,
                                       int64_t C, int32_t iters, const rodinia_hotspot_coeffs* c) {
    if (!tin || !p || !tout) return set_error(RODINIA_E_INVALID, "hotspot: null buffer");
    if (R < 1 || C < 1) return set_error(RODINIA_E_INVALID, "hotspot: rows/cols must be >= 1");
    if (R > (1ll << 31) - 1 || C > (1ll << 31) - 1 || R * C > (1ll << 40))
        return set_error(RODINIA_E_INVALID, "hotspot: grid too large");
    if (iters < 0) return set_error(RODINIA_E_INVALID, "hotspot: iterations < 0");
    if (tin == tout) return set_error(RODINIA_E_INVALID, "hotspot: temp_out must not alias temp_in");
    if (c && !(std::isfinite(c->k) && std::isfinite(c->rx) && std::isfinite(c->ry) &&
               std::isfinite(c->rz) && std::isfinite(c->amb)))
        return set_error(RODINIA_E_INVALID, "hotspot: coefficients must be finite");
    return RODINIA_OK;
}

static rodinia_status hotspot_resolve(int64_t R, int64_t C, int32_t iters, const rodinia_granularity* g,
                                      rodinia_granularity* out) {
    if (!gran_is_zero(g)) { *out = *g; return RODINIA_OK; }
    rodinia_problem pb{R, C, iters, 1};
    if (tune_cache_lookup(RODINIA_HOTSPOT, pb, out)) return RODINIA_OK;
    *out = default_gran(RODINIA_HOTSPOT, pb);
    return RODINIA_OK;
}

extern "C" rodinia_status rodinia_hotspot(const float* tin, const float* p, float* tout, float* scratch,
                                          int64_t R, int64_t C, int32_t iters,
                                          const rodinia_hotspot_coeffs* coeffs,
                                          const rodinia_granularity* g, void* stream) {
    RG_TRY(hotspot_validate(tin, p, tout, R, C, iters, coeffs));
    if (scratch && (scratch == tin || scratch == tout))
        return set_error(RODINIA_E_INVALID, "hotspot: scratch aliases an operand");
    rodinia_granularity gg;
    RG_TRY(hotspot_resolve(R, C, iters, g, &gg));
    const hotspot::DirectVariant* dv;
    const hotspot::StreamVariant* sv;
    RG_TRY(hotspot::check(gg, R, C, &dv, &sv));
    rodinia_hotspot_coeffs cc;
    if (coeffs) cc = *coeffs;
    else rodinia_hotspot_coeffs_rodinia(R, C, 0.016, 0.016, &cc);
    DeviceInfo di;
    RG_TRY(device_info(&di));
    cudaStream_t s = (cudaStream_t)stream;
    float* scr = scratch;
    float* kp = nullptr;
    const size_t bytes = (size_t)R * C * sizeof(float);
    if (!scr && iters >= 1) RG_TRY(scratch_alloc((void**)&scr, bytes, s));
    rodinia_status st = RODINIA_OK;
    if (iters >= 1) st = scratch_alloc((void**)&kp, bytes, s);
    if (st == RODINIA_OK) st = hotspot::solve(tin, p, tout, scr, kp, (int)R, (int)C, iters, cc, gg, dv, sv, s);
    if (kp) scratch_free(kp, s);
    if (scr != scratch) scratch_free(scr, s);
    return st;
}

// Cached device buffers for the *_host entry points (grown on demand, per process).
namespace rg {
struct HostStage {
    std::mutex mu;
    void* buf[9] = {nullptr};   // 0..2: *_host calls; 3..8: two buffer sets of the batch call
    size_t cap[9] = {0};
    int dev[9] = {-1, -1, -1, -1, -1, -1, -1, -1, -1};
    cudaStream_t h2d = nullptr, d2h = nullptr;  // copy streams of rodinia_hotspot_host_batch
    cudaEvent_t ev[6] = {nullptr};              // per set: inputs landed, solved, result read
    int sdev = -1;
};
HostStage& host_stage() {
    static HostStage hs;
    return hs;
}
std::mutex& host_mutex() { return host_stage().mu; }
rodinia_status host_buffer(int i, size_t bytes, void** out) {
    HostStage& hs = host_stage();
    int dev = 0;
    RG_CUDA(cudaGetDevice(&dev));
    if (hs.cap[i] < bytes || hs.dev[i] != dev) {
        if (hs.buf[i]) cudaFree(hs.buf[i]);
        hs.buf[i] = nullptr;
        hs.cap[i] = 0;
        RG_CUDA(cudaMalloc(&hs.buf[i], bytes));
        hs.cap[i] = bytes;
        hs.dev[i] = dev;
    }
    *out = hs.buf[i];
    return RODINIA_OK;
}
}  // namespace rg

extern "C" rodinia_status rodinia_hotspot_host(const float* tin, const float* p, float* tout, int64_t R,
                                               int64_t C, int32_t iters,
                                               const rodinia_hotspot_coeffs* coeffs,
                                               const rodinia_granularity* g, void* stream) {
    RG_TRY(hotspot_validate(tin, p, tout, R, C, iters, coeffs));
    DeviceInfo di;
    RG_TRY(device_info(&di));
    std::lock_guard<std::mutex> lk(host_stage().mu);
    const size_t bytes = (size_t)R * C * sizeof(float);
    void *dt, *dp, *dout;
    RG_TRY(host_buffer(0, bytes, &dt));
    RG_TRY(host_buffer(1, bytes, &dp));
    RG_TRY(host_buffer(2, bytes, &dout));
    cudaStream_t s = (cudaStream_t)stream;
    RG_CUDA(cudaMemcpyAsync(dt, tin, bytes, cudaMemcpyHostToDevice, s));
    RG_CUDA(cudaMemcpyAsync(dp, p, bytes, cudaMemcpyHostToDevice, s));
    RG_TRY(rodinia_hotspot((const float*)dt, (const float*)dp, (float*)dout, nullptr, R, C, iters, coeffs, g, stream));
    RG_CUDA(cudaMemcpyAsync(tout, dout, bytes, cudaMemcpyDeviceToHost, s));
    RG_CUDA(cudaStreamSynchronize(s));
    return RODINIA_OK;
}

extern "C" rodinia_status rodinia_hotspot_host_batch(const float* const* tin, const float* const* p,
                                                     float* const* tout, int32_t count, int64_t R, int64_t C,
                                                     int32_t iters, const rodinia_hotspot_coeffs* coeffs,
                                                     const rodinia_granularity* g, void* stream) {
    if (count < 0 || (count > 0 && (!tin || !p || !tout)))
        return set_error(RODINIA_E_INVALID, "hotspot_host_batch: bad arguments");
    for (int i = 0; i < count; ++i) RG_TRY(hotspot_validate(tin[i], p[i], tout[i], R, C, iters, coeffs));
    if (count == 0) return RODINIA_OK;
    DeviceInfo di;
    RG_TRY(device_info(&di));
    HostStage& hs = host_stage();
    std::lock_guard<std::mutex> lk(hs.mu);
    if (hs.sdev != di.device) {
        RG_CUDA(cudaStreamCreateWithFlags(&hs.h2d, cudaStreamNonBlocking));
        RG_CUDA(cudaStreamCreateWithFlags(&hs.d2h, cudaStreamNonBlocking));
        for (auto& e : hs.ev) RG_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        hs.sdev = di.device;
    }
    const size_t bytes = (size_t)R * C * sizeof(float);
    void* dv[2][3];
    for (int b = 0; b < 2; ++b)
        for (int k = 0; k < 3; ++k) RG_TRY(host_buffer(3 + 3 * b + k, bytes, &dv[b][k]));
    cudaStream_t s = (cudaStream_t)stream;
    cudaEvent_t* in_ready = hs.ev;        // [2]: H2D of the set's inputs done
    cudaEvent_t* solved = hs.ev + 2;      // [2]: solve done (inputs free, output valid)
    cudaEvent_t* read = hs.ev + 4;        // [2]: D2H of the set's output done
    auto h2d = [&](int i) -> rodinia_status {
        const int b = i & 1;
        if (i >= 2) RG_CUDA(cudaStreamWaitEvent(hs.h2d, solved[b], 0));  // problem i-2 done with the set
        RG_CUDA(cudaMemcpyAsync(dv[b][0], tin[i], bytes, cudaMemcpyHostToDevice, hs.h2d));
        RG_CUDA(cudaMemcpyAsync(dv[b][1], p[i], bytes, cudaMemcpyHostToDevice, hs.h2d));
        RG_CUDA(cudaEventRecord(in_ready[b], hs.h2d));
        return RODINIA_OK;
    };
    RG_TRY(h2d(0));
    for (int i = 0; i < count; ++i) {
        const int b = i & 1;
        if (i + 1 < count) RG_TRY(h2d(i + 1));  // next inputs stream in while problem i solves
        RG_CUDA(cudaStreamWaitEvent(s, in_ready[b], 0));
        if (i >= 2) RG_CUDA(cudaStreamWaitEvent(s, read[b], 0));  // output of problem i-2 read back
        RG_TRY(rodinia_hotspot((const float*)dv[b][0], (const float*)dv[b][1], (float*)dv[b][2], nullptr, R, C, iters,
                               coeffs, g, stream));
        RG_CUDA(cudaEventRecord(solved[b], s));
        RG_CUDA(cudaStreamWaitEvent(hs.d2h, solved[b], 0));  // result of problem i streams out
        RG_CUDA(cudaMemcpyAsync(tout[i], dv[b][2], bytes, cudaMemcpyDeviceToHost, hs.d2h));
        RG_CUDA(cudaEventRecord(read[b], hs.d2h));
    }
    RG_CUDA(cudaStreamSynchronize(hs.d2h));
    RG_CUDA(cudaStreamSynchronize(s));
    return RODINIA_OK;
}

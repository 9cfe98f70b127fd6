// tune.cu -- variant enumeration with the compile-time (ptxas) filter, and the timing-driven
// tuner (TDO): every surviving alternative is run on synthetic data of the
// problem's shape, timed with CUDA events (one warm-up, `reps` timed runs, median), the
// fastest is returned and cached.
#include <cuda_runtime.h>
#include <string.h>

#include <algorithm>
#include <vector>

#include "hs_cell.cuh"
#include "workloads.h"
#include "rg_internal.h"

namespace rg {

extern const PtxasStats kPtxasStats[];
extern const int kNumPtxasStats;

float model_estimate_ms(rodinia_kernel k, const rodinia_problem& p, const rodinia_tune_row& row);  // model.cu

const PtxasStats* find_stats(const char* key) {
    for (int i = 0; i < kNumPtxasStats; ++i)
        if (strcmp(kPtxasStats[i].key, key) == 0) return &kPtxasStats[i];
    return nullptr;
}

// ---------------------------------------------------------------- per-workload registries
namespace hotspot {
struct DirectVariant;
struct StreamVariant;
int num_variants();
void variant_info(int i, rodinia_granularity* g, const void** fn, const char** key, int* threads);
}  // namespace hotspot

struct Registry {
    int (*count)();
    void (*info)(int, rodinia_granularity*, const void**, const char**, int*);
};

// Filled in by the other workload TUs through these hooks.
int srad_num_variants();
void srad_variant_info(int, rodinia_granularity*, const void**, const char**, int*);
int pathfinder_num_variants();
void pathfinder_variant_info(int, rodinia_granularity*, const void**, const char**, int*);
int lud_num_variants();
void lud_variant_info(int, rodinia_granularity*, const void**, const char**, int*);
int hotspot3d_num_variants();
void hotspot3d_variant_info(int, rodinia_granularity*, const void**, const char**, int*);

static Registry registry(rodinia_kernel k) {
    switch (k) {
        case RODINIA_HOTSPOT: return {hotspot::num_variants, hotspot::variant_info};
        case RODINIA_SRAD: return {srad_num_variants, srad_variant_info};
        case RODINIA_PATHFINDER: return {pathfinder_num_variants, pathfinder_variant_info};
        case RODINIA_LUD: return {lud_num_variants, lud_variant_info};
        case RODINIA_HOTSPOT3D: return {hotspot3d_num_variants, hotspot3d_variant_info};
    }
    return {nullptr, nullptr};
}

static void fill_row(rodinia_kernel k, int i, bool have_dev, int base_spill, rodinia_tune_row* r) {
    Registry reg = registry(k);
    const void* fn;
    const char* key;
    int threads;
    memset(r, 0, sizeof *r);
    reg.info(i, &r->g, &fn, &key, &threads);
    const PtxasStats* st = find_stats(key);
    r->median_ms = -1.0f;
    r->model_ms = -1.0f;
    r->regs = st ? st->regs : -1;
    r->spill_bytes = st ? st->spill_stores + st->spill_loads : -1;
    r->smem_bytes = st ? st->smem : -1;
    r->threads = threads;
    r->ctas_per_sm = have_dev ? ctas_per_sm(fn, threads, 0) : 0;
    r->status = filter_decision(st, threads, 0, base_spill);
    if (r->status == RODINIA_OK && have_dev && r->ctas_per_sm == 0) r->status = RODINIA_E_FILTERED;
}

static int family_base_spill(rodinia_kernel k) {
    // The uncoarsened kernel of each workload is variant 0 of its registry.
    Registry reg = registry(k);
    if (reg.count() == 0) return 0;
    rodinia_granularity g;
    const void* fn;
    const char* key;
    int threads;
    reg.info(0, &g, &fn, &key, &threads);
    const PtxasStats* st = find_stats(key);
    return st ? st->spill_stores + st->spill_loads : 0;
}

// The compile-time filter at the boundary: an explicitly requested
// instantiation the ptxas filter prunes is refused with RODINIA_E_FILTERED (host-only, before
// any launch) unless the caller sets RODINIA_FORCE.  Same decision as rodinia_variants().
rodinia_status boundary_filter(rodinia_kernel k, const char* key, int threads, int dyn_smem, int flags) {
    if (flags & RODINIA_FORCE) return RODINIA_OK;
    static int base[5] = {-1, -1, -1, -1, -1};
    const int ki = (int)k;
    if (ki < 0 || ki >= 5) return RODINIA_OK;
    if (base[ki] < 0) base[ki] = family_base_spill(k);
    const PtxasStats* st = find_stats(key);
    const rodinia_status s = filter_decision(st, threads, dyn_smem, base[ki]);
    if (s == RODINIA_OK) return RODINIA_OK;
    return set_error(s, "%s is pruned by the compile-time filter (%d registers, %d B spill stores + %d B "
                        "loads, %d B shared memory, %d threads; PAPER.md:267); set RODINIA_FORCE to run it",
                     key, st ? st->regs : -1, st ? st->spill_stores : -1, st ? st->spill_loads : -1,
                     (st ? st->smem : 0) + dyn_smem, threads);
}

rodinia_granularity default_gran(rodinia_kernel k, const rodinia_problem& p) {
    switch (k) {
        case RODINIA_HOTSPOT:
            // B200 default (measured on 16384^2): streaming temporal blocking,
            // 4 columns per lane, 8 steps per launch, 1 band per CTA, 128-row chunks,
            // register budget for 12 CTAs/SM.
            if (p.iterations >= 8 && p.cols >= 128) return gran(4, 1, 1, 8, 8, 1, RODINIA_STREAM | RODINIA_OCC(12));
            return gran(4, 1, 1, 1, 1, 1);
        case RODINIA_SRAD: return gran(4, 1, 1, 2, 1, 1, RODINIA_STREAM);
        case RODINIA_PATHFINDER: return gran(4, 1, 1, 1, 8, 1);
        case RODINIA_HOTSPOT3D: return gran(4, 1, 1, 1, 1, 1);
        case RODINIA_LUD:  // measured on B200 at n = 8192
            return p.iterations == 32 ? gran(2, 4, 4, 2, 1, 1) : gran(4, 2, 2, 2, 1, 1);
    }
    return gran(1, 1, 1, 1, 1, 0);
}

// ---------------------------------------------------------------- pre-pruning gate
// rodinia_tune_pruned runs a workload's tuner twice: a collect pass in which every candidate
// that survives the compile-time filter is recorded with its model estimate and not timed, and
// a select pass in which only the `keep` best-estimated candidates (and every candidate the
// model cannot estimate) are timed.  Tuners call prune_gate() between the filter and timing.
namespace {
struct PruneState {
    bool active = false, collect = false;
    std::vector<rodinia_tune_row> seen;
    std::vector<rodinia_granularity> keep;
};
thread_local PruneState g_prune;
bool same_gran(const rodinia_granularity& a, const rodinia_granularity& b) { return memcmp(&a, &b, sizeof a) == 0; }
}  // namespace

bool prune_active() { return g_prune.active; }

rodinia_status prune_gate(rodinia_kernel k, const rodinia_problem& p, rodinia_tune_row* row) {
    row->model_ms = model_estimate_ms(k, p, *row);
    if (!g_prune.active) return RODINIA_OK;
    if (g_prune.collect) {
        g_prune.seen.push_back(*row);
        return RODINIA_E_PRUNED;
    }
    if (row->model_ms < 0) return RODINIA_OK;
    for (const auto& g : g_prune.keep)
        if (same_gran(g, row->g)) return RODINIA_OK;
    return RODINIA_E_PRUNED;
}

// ---------------------------------------------------------------- synthetic data
__global__ void rg_fill(float* a, int64_t n, float base, float scale, uint32_t seed) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        uint32_t x = (uint32_t)i * 2654435761u ^ seed;
        x ^= x >> 13; x *= 0x5bd1e995u; x ^= x >> 15;
        a[i] = base + scale * (float)(x & 0xffffff) * (1.0f / 16777216.0f);
    }
}

static rodinia_status fill(float* a, int64_t n, float base, float scale, uint32_t seed, cudaStream_t s) {
    rg_fill<<<1184, 256, 0, s>>>(a, n, base, scale, seed);
    RG_CUDA(cudaGetLastError());
    return RODINIA_OK;
}

// Candidate granularities for hotspot, two stages (DESIGN.md §5 "TDO"):
//  stage 1: every instantiation with its base block factors;
//  stage 2: the 4 fastest instantiations of stage 1 with a sweep of block factors (any
//           integer is legal; primes included on purpose).
static void hotspot_stage1(std::vector<rodinia_granularity>* out) {
    const int n = hotspot::num_variants();
    for (int i = 0; i < n; ++i) {
        rodinia_granularity g;
        const void* fn;
        const char* key;
        int threads;
        hotspot::variant_info(i, &g, &fn, &key, &threads);
        if (g.flags & RODINIA_STREAM) {
            g.block_x = 1; g.block_y = 4; out->push_back(g);
            g.block_y = 8; out->push_back(g);
        } else {
            g.block_x = 1; g.block_y = 1; out->push_back(g);
            g.block_x = 2; out->push_back(g);
        }
    }
}

// Stage 2: block factors of one instantiation.  For the stream family the chunk height also gets
// "wave-fitted" candidates: with S resident CTAs per wave (occupancy x SMs) and B bands, chunks
// such that B x chunks fills w whole waves (w = 1..4, 8, 9) -- the fixed list alone leaves a
// partial last wave on slab shapes (2048-row slabs at 8 ranks: 2.2 waves at by = 6).
static void hotspot_stage2(const rodinia_granularity& base, int64_t R, int64_t C, std::vector<rodinia_granularity>* out) {
    rodinia_granularity g = base;
    if (g.flags & RODINIA_STREAM) {
        std::vector<int> bys = {2, 3, 4, 6, 8, 12, 16, 24};
        const int n = hotspot::num_variants();
        int slots = 0;
        for (int i = 0; i < n; ++i) {
            rodinia_granularity vg;
            const void* fn;
            const char* key;
            int threads;
            hotspot::variant_info(i, &vg, &fn, &key, &threads);
            if (vg.thread_x == g.thread_x && vg.temporal == g.temporal && vg.flags == g.flags) {
                DeviceInfo di;
                if (device_info(&di) == RODINIA_OK) slots = ctas_per_sm(fn, threads, 0) * di.sms;
                break;
            }
        }
        const int ow = 32 * g.thread_x - 2 * g.temporal;
        const int64_t bands = ow > 0 ? (C + ow - 1) / ow : 0;
        if (slots > 0 && bands > 0 && bands <= slots) {
            for (int w : {1, 2, 3, 4, 8, 9}) {
                const int64_t chunks = (int64_t)w * (slots / bands);
                const int64_t by = (R + 16 * chunks - 1) / (16 * chunks);
                if (by >= 1 && by <= 256 && std::find(bys.begin(), bys.end(), (int)by) == bys.end()) bys.push_back((int)by);
            }
        }
        for (int bx : {1, 2})
            for (int by : bys) { g.block_x = bx; g.block_y = by; out->push_back(g); }
    } else {
        static const int bxy[][2] = {{1, 1}, {2, 1}, {3, 1}, {4, 1}, {7, 1}, {1, 2}, {2, 2}, {4, 4}};
        for (auto& b : bxy) { g.block_x = b[0]; g.block_y = b[1]; out->push_back(g); }
    }
}

static bool same_instantiation(const rodinia_granularity& a, const rodinia_granularity& b) {
    return a.thread_x == b.thread_x && a.thread_y == b.thread_y && a.temporal == b.temporal &&
           a.index_mode == b.index_mode && a.flags == b.flags;
}

static float median(std::vector<float> v) {
    std::sort(v.begin(), v.end());
    return v.empty() ? -1.f : v[v.size() / 2];
}

static rodinia_status tune_hotspot(const rodinia_problem& p, int reps, rodinia_granularity* best,
                                   std::vector<rodinia_tune_row>* rows) {
    const int64_t R = p.rows, C = p.cols;
    const int iters = std::max(1, std::min(p.iterations, 24));
    cudaStream_t s;
    RG_CUDA(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    float *tin = nullptr, *pw = nullptr, *tout = nullptr, *scr = nullptr;
    const size_t bytes = (size_t)R * C * sizeof(float);
    rodinia_status st = RODINIA_OK;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    if (cudaMalloc(&tin, bytes) != cudaSuccess || cudaMalloc(&pw, bytes) != cudaSuccess ||
        cudaMalloc(&tout, bytes) != cudaSuccess || cudaMalloc(&scr, bytes) != cudaSuccess) {
        cudaGetLastError();
        st = set_error(RODINIA_E_NOMEM, "tune: cannot allocate %zu-byte buffers", bytes);
    }
    // states u = T - amb and pre-scaled power kP = k*P of the synthetic recipe (hs_cell.cuh);
    // the stepping kernels' run time does not depend on the values
    rodinia_hotspot_coeffs cc;
    rodinia_hotspot_coeffs_rodinia(R, C, R * 31.25e-6, C * 31.25e-6, &cc);
    const HsCoef cf = hs_derive(cc.k, cc.rx, cc.ry, cc.rz);
    if (st == RODINIA_OK) st = fill(tin, R * C, 323.15f - cc.amb, 20.0f, 1u, s);
    if (st == RODINIA_OK) st = fill(pw, R * C, 0.0f, 1e-3f * cc.k, 2u, s);
    const int base_spill = family_base_spill(RODINIA_HOTSPOT);
    float best_ms = 1e30f;
    auto time_one = [&](const rodinia_granularity& gc) {
        rodinia_tune_row row;
        memset(&row, 0, sizeof row);
        row.g = gc;
        row.median_ms = -1.f;
        row.model_ms = -1.f;
        const hotspot::DirectVariant* dv;
        const hotspot::StreamVariant* sv;
        rodinia_status cs = hotspot::check(row.g, R, C, &dv, &sv);
        if (cs == RODINIA_OK) {
            const int n = hotspot::num_variants();
            for (int i = 0; i < n; ++i) {
                rodinia_granularity g;
                const void* fn;
                const char* key;
                int threads;
                hotspot::variant_info(i, &g, &fn, &key, &threads);
                if (same_instantiation(g, row.g)) {
                    const PtxasStats* ps = find_stats(key);
                    row.regs = ps ? ps->regs : -1;
                    row.spill_bytes = ps ? ps->spill_stores + ps->spill_loads : -1;
                    row.smem_bytes = ps ? ps->smem : -1;
                    row.threads = threads;
                    row.ctas_per_sm = ctas_per_sm(fn, threads, 0);
                    cs = filter_decision(ps, threads, 0, base_spill);
                    if (cs == RODINIA_OK && row.ctas_per_sm == 0) cs = RODINIA_E_FILTERED;
                    break;
                }
            }
        }
        if (cs == RODINIA_OK) cs = prune_gate(RODINIA_HOTSPOT, p, &row);
        if (cs == RODINIA_OK) {
            std::vector<float> ts;
            for (int r = -1; r < reps && cs == RODINIA_OK; ++r) {
                cudaEventRecord(e0, s);
                cs = hotspot::run(tin, pw, tout, scr, (int)R, (int)C, iters, cf, row.g, dv, sv, s);
                cudaEventRecord(e1, s);
                if (cudaEventSynchronize(e1) != cudaSuccess) {
                    cs = cuda_error(cudaGetLastError(), "tune run", __FILE__, __LINE__);
                    st = cs;  // a faulting variant is a hard error
                }
                float ms = 0;
                cudaEventElapsedTime(&ms, e0, e1);
                if (r >= 0) ts.push_back(ms);
            }
            if (cs == RODINIA_OK) {
                row.median_ms = median(ts);
                if (row.median_ms < best_ms) { best_ms = row.median_ms; *best = row.g; }
            }
        }
        row.status = cs;
        rows->push_back(row);
    };
    std::vector<rodinia_granularity> stage1;
    hotspot_stage1(&stage1);
    for (size_t i = 0; st == RODINIA_OK && i < stage1.size(); ++i) time_one(stage1[i]);
    // stage 2: best 4 distinct instantiations
    std::vector<rodinia_tune_row> ok;
    for (auto& r : *rows) if (r.status == RODINIA_OK && r.median_ms > 0) ok.push_back(r);
    std::sort(ok.begin(), ok.end(), [](const rodinia_tune_row& a, const rodinia_tune_row& b) { return a.median_ms < b.median_ms; });
    std::vector<rodinia_granularity> tops;
    if (prune_active()) {
        // pre-pruning: the model ranks the block-factor sweep of every instantiation
        for (auto& g : stage1) {
            bool dup = false;
            for (auto& t : tops) dup = dup || same_instantiation(t, g);
            if (!dup) tops.push_back(g);
        }
        ok.clear();
    }
    for (auto& r : ok) {
        bool dup = false;
        for (auto& t : tops) dup = dup || same_instantiation(t, r.g);
        if (!dup) tops.push_back(r.g);
        if (tops.size() == 4) break;
    }
    for (auto& t : tops) {
        std::vector<rodinia_granularity> stage2;
        hotspot_stage2(t, R, C, &stage2);
        for (auto& g : stage2) {
            bool seen = false;
            for (auto& r : *rows) seen = seen || (memcmp(&r.g, &g, sizeof g) == 0);
            if (!seen && st == RODINIA_OK) time_one(g);
        }
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(tin); cudaFree(pw); cudaFree(tout); cudaFree(scr);
    cudaStreamDestroy(s);
    if (st == RODINIA_OK && best_ms >= 1e29f) st = set_error(RODINIA_E_FILTERED, "tune: no variant survived");
    if (st == RODINIA_OK) tune_cache_store(RODINIA_HOTSPOT, p, *best, best_ms);
    return st;
}

rodinia_status tune_srad(const rodinia_problem& p, int reps, rodinia_granularity* best, std::vector<rodinia_tune_row>* rows);
rodinia_status tune_pathfinder(const rodinia_problem& p, int reps, rodinia_granularity* best, std::vector<rodinia_tune_row>* rows);
rodinia_status tune_lud(const rodinia_problem& p, int reps, rodinia_granularity* best, std::vector<rodinia_tune_row>* rows);
rodinia_status tune_hotspot3d(const rodinia_problem& p, int reps, rodinia_granularity* best, std::vector<rodinia_tune_row>* rows);

}  // namespace rg

using namespace rg;

extern "C" rodinia_status rodinia_variants(rodinia_kernel k, rodinia_tune_row* out, int32_t* n) {
    if (!n || *n < 0 || (*n > 0 && !out)) return set_error(RODINIA_E_INVALID, "variants: bad arguments");
    if ((int)k < 0 || (int)k > 4) return set_error(RODINIA_E_INVALID, "variants: unknown kernel %d", (int)k);
    Registry reg = registry(k);
    const int total = reg.count();
    int cnt = 0;
    cudaGetDeviceCount(&cnt);
    cudaGetLastError();
    const bool have_dev = cnt > 0;
    const int base_spill = family_base_spill(k);
    for (int i = 0; i < total && i < *n; ++i) fill_row(k, i, have_dev, base_spill, &out[i]);
    *n = total;
    return RODINIA_OK;
}

extern "C" rodinia_status rodinia_tune(rodinia_kernel k, const rodinia_problem* p, int32_t reps,
                                       rodinia_granularity* best, rodinia_tune_row* rows, int32_t* nrows) {
    if (!p || !best || reps < 1 || p->rows < 1 || p->cols < 1 || p->iterations < 0 || p->nranks < 1)
        return set_error(RODINIA_E_INVALID, "tune: bad arguments");
    if (nrows && *nrows > 0 && !rows) return set_error(RODINIA_E_INVALID, "tune: rows is null");
    if ((int)k < 0 || (int)k > 4) return set_error(RODINIA_E_INVALID, "tune: unknown kernel %d", (int)k);
    DeviceInfo di;
    RG_TRY(device_info(&di));
    std::vector<rodinia_tune_row> out;
    rodinia_status st;
    switch (k) {
        case RODINIA_HOTSPOT: st = tune_hotspot(*p, reps, best, &out); break;
        case RODINIA_SRAD: st = tune_srad(*p, reps, best, &out); break;
        case RODINIA_PATHFINDER: st = tune_pathfinder(*p, reps, best, &out); break;
        case RODINIA_HOTSPOT3D: st = tune_hotspot3d(*p, reps, best, &out); break;
        default: st = tune_lud(*p, reps, best, &out); break;
    }
    if (nrows) {
        const int cap = *nrows;
        for (int i = 0; i < cap && i < (int)out.size(); ++i) rows[i] = out[i];
        *nrows = (int)out.size();
    }
    return st;
}

static rodinia_status run_tuner(rodinia_kernel k, const rodinia_problem& p, int reps, rodinia_granularity* best,
                                std::vector<rodinia_tune_row>* out) {
    switch (k) {
        case RODINIA_HOTSPOT: return tune_hotspot(p, reps, best, out);
        case RODINIA_SRAD: return tune_srad(p, reps, best, out);
        case RODINIA_PATHFINDER: return tune_pathfinder(p, reps, best, out);
        case RODINIA_HOTSPOT3D: return tune_hotspot3d(p, reps, best, out);
        default: return tune_lud(p, reps, best, out);
    }
}

extern "C" rodinia_status rodinia_tune_pruned(rodinia_kernel k, const rodinia_problem* p, int32_t reps, int32_t keep,
                                              rodinia_granularity* best, rodinia_tune_row* rows, int32_t* nrows) {
    if (keep <= 0) return rodinia_tune(k, p, reps, best, rows, nrows);
    if (!p || !best || reps < 1 || p->rows < 1 || p->cols < 1 || p->iterations < 0 || p->nranks < 1)
        return set_error(RODINIA_E_INVALID, "tune_pruned: bad arguments");
    if (nrows && *nrows > 0 && !rows) return set_error(RODINIA_E_INVALID, "tune_pruned: rows is null");
    if ((int)k < 0 || (int)k > 4) return set_error(RODINIA_E_INVALID, "tune_pruned: unknown kernel %d", (int)k);
    DeviceInfo di;
    RG_TRY(device_info(&di));
    // collect pass: every filter survivor with its model estimate, nothing timed
    g_prune = PruneState();
    g_prune.active = true;
    g_prune.collect = true;
    std::vector<rodinia_tune_row> scratch;
    rodinia_granularity dummy;
    rodinia_status st = run_tuner(k, *p, reps, &dummy, &scratch);
    if (st != RODINIA_OK && st != RODINIA_E_FILTERED) {
        g_prune = PruneState();
        return st;
    }
    clear_error();
    std::vector<rodinia_tune_row> ranked;
    for (auto& r : g_prune.seen)
        if (r.model_ms >= 0) ranked.push_back(r);
    std::stable_sort(ranked.begin(), ranked.end(),
                     [](const rodinia_tune_row& a, const rodinia_tune_row& b) { return a.model_ms < b.model_ms; });
    for (size_t i = 0; i < ranked.size() && (int)g_prune.keep.size() < keep; ++i) {
        bool dup = false;
        for (auto& g : g_prune.keep) dup = dup || same_gran(g, ranked[i].g);
        if (!dup) g_prune.keep.push_back(ranked[i].g);
    }
    // select pass: time the kept candidates (and every unmodelled one)
    g_prune.collect = false;
    std::vector<rodinia_tune_row> out;
    st = run_tuner(k, *p, reps, best, &out);
    g_prune = PruneState();
    if (nrows) {
        const int cap = *nrows;
        for (int i = 0; i < cap && i < (int)out.size(); ++i) rows[i] = out[i];
        *nrows = (int)out.size();
    }
    return st;
}

extern "C" rodinia_status rodinia_resolve(rodinia_kernel k, const rodinia_problem* p, rodinia_granularity* out) {
    if (!p || !out) return set_error(RODINIA_E_INVALID, "resolve: bad arguments");
    if (tune_cache_lookup(k, *p, out)) return RODINIA_OK;
    *out = default_gran(k, *p);
    return RODINIA_OK;
}

extern "C" rodinia_status rodinia_split_total(int32_t total, int32_t ndims, int32_t out[3]) {
    if (!out || total < 1 || ndims < 1 || ndims > 3) return set_error(RODINIA_E_INVALID, "split_total: bad arguments");
    std::vector<int> primes;
    int t = total;
    for (int p = 2; (int64_t)p * p <= t; ++p)
        while (t % p == 0) { primes.push_back(p); t /= p; }
    if (t > 1) primes.push_back(t);
    std::sort(primes.rbegin(), primes.rend());
    int f[3] = {1, 1, 1};
    for (int p : primes) {
        int best = 0;
        for (int d = 1; d < ndims; ++d)
            if (f[d] < f[best]) best = d;
        f[best] *= p;
    }
    for (int d = 0; d < 3; ++d) out[d] = f[d];
    return RODINIA_OK;
}

// dist.cu -- multi-GPU row-slab decomposition for the stencils (hotspot, srad), one process
// per GPU, NCCL point-to-point halo exchange over NVLink / NVSwitch (SURVEY §8(e)
// and §8(a) S13).
//
// Rank r owns global rows [floor(r*R/P), floor((r+1)*R/P)).  Its local buffer is
//   [top halo][own rows][bottom halo]
// and the kernels clamp neighbours at the *buffer* edges, so the same launch code as the
// single-GPU path runs on a slab: rows next to a non-global buffer edge go stale by one row
// (hotspot; srad: one row at the top, two at the bottom) per step, which the halo depth absorbs.
//  * hotspot: halo D = steps fused per launch (temporal); every D steps each rank sends its
//    first D own rows up and its last D own rows down (ncclSend/ncclRecv in one group).  The
//    exchange overlaps the interior launch: the owned rows alone determine output rows
//    [D, own-D) after D steps, so the interior runs on the compute stream while a side stream
//    exchanges the halos and then computes the two boundary strips (D halo rows + 2D owned rows
//    each) into strip buffers; the compute stream copies their D valid rows in after the
//    interior.  Power halos are exchanged once per call.
//  * srad: one iteration reads rows i-1..i+2, so halos are D above and 2D below, exchanged
//    every D iterations (D = the granularity's temporal depth; default min(8, own/2)).  The
//    global ROI statistics q0sqr(t) are computed without any per-iteration collective: every
//    rank gathers the ROI's dependency cone of J0 once (rows [r1-n, r2+2n+2] x cols likewise,
//    ncclBroadcast from the owners) and evolves just that window with the same kernels; ROI
//    values on the window are bit-identical to the full grid (reading S10), hence so is q0sqr(t).
// Results are bitwise identical to the single-GPU call with the same granularity.  The slab
// buffers, strip buffers, srad engines and the side stream live in the communicator and are
// reused by later calls of the same shape (no per-call allocation after the first).
//
// A second communicator kind, LOCAL, keeps all P slabs on the current device and moves halos
// with cudaMemcpyAsync; it runs the identical slab/halo/overlap logic on one GPU (tests).
//
// NCCL is not linked: libnccl.so.2 is dlopen'ed at run time (the copy torch already mapped,
// or $RODINIA_NCCL_LIB), so the library loads on hosts without NCCL.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>  // types and enum values only; entry points are resolved with dlsym
#include <string.h>

#include <algorithm>
#include <cmath>
#include <mutex>
#include <vector>

#include "rg_internal.h"
#include "workloads.h"

namespace rg {
struct Slab {
    int rank;       // global slab index
    int64_t row0;   // first owned global row
    int own;        // owned rows
    int top, bot;   // halo rows above / below
    float* buf[2];  // local buffers (top + own + bot rows)
    float* aux;     // hotspot: pre-scaled power kP; unused for srad
    float* scr;     // hotspot: ping-pong scratch for multi-launch periods
    float* strip[2];     // hotspot overlap: boundary-strip outputs (top, bottom), 3D rows each
    float* strip_scr;    // ... and their ping-pong scratch
    int rows() const { return top + own + bot; }
};
namespace srad { struct Engine; }
}  // namespace rg

struct rodinia_comm {
    int kind;  // 0 = NCCL (one slab per process), 1 = LOCAL (all slabs in this process)
    int nranks, rank;
    ncclComm_t nccl;
    std::mutex mu;
    int dev = -1;
    cudaStream_t side = nullptr;          // exchange + boundary strips (hotspot overlap)
    cudaEvent_t ev_ready = nullptr, ev_strips = nullptr;
    cudaEvent_t ev_done = nullptr;        // end of the previous call (orders calls on any stream)
    bool done_recorded = false;
    std::vector<cudaEvent_t> ev_cone;     // srad: q0sqr of exchange period p is ready
    // persistent buffers of the last shape (hotspot and srad separately)
    struct HsCache { int64_t R = 0, C = 0; int D = 0; std::vector<rg::Slab> sl; } hs;
    struct SrCache {
        int64_t R = 0, C = 0; int D = 0, niter_cap = 0, WR = 0, WC = 0;
        rodinia_granularity g{};
        std::vector<rg::Slab> sl;
        std::vector<rg::srad::Engine> eng;
        rg::srad::Engine we;
        float* W = nullptr;
        bool have_we = false;
    } sr;
};

namespace rg {

// ------------------------------------------------------------------ NCCL loader
struct NcclApi {
    bool ok = false;
    ncclResult_t (*GetUniqueId)(ncclUniqueId*);
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int);
    ncclResult_t (*CommDestroy)(ncclComm_t);
    ncclResult_t (*CommGetAsyncError)(ncclComm_t, ncclResult_t*);
    ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t);
    ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t);
    ncclResult_t (*Bcast)(const void*, void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t);
    ncclResult_t (*GroupStart)();
    ncclResult_t (*GroupEnd)();
    const char* (*GetErrorString)(ncclResult_t);
};

static rodinia_status nccl_api(NcclApi** out) {
    static std::mutex mu;
    static NcclApi api;
    static bool tried = false;
    std::lock_guard<std::mutex> lk(mu);
    if (!tried) {
        tried = true;
        const char* env = getenv("RODINIA_NCCL_LIB");
        void* h = nullptr;
        if (env && *env) h = dlopen(env, RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
        if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (h) {
#define RG_SYM(f, n) api.f = (decltype(api.f))dlsym(h, n)
            RG_SYM(GetUniqueId, "ncclGetUniqueId");
            RG_SYM(CommInitRank, "ncclCommInitRank");
            RG_SYM(CommDestroy, "ncclCommDestroy");
            RG_SYM(CommGetAsyncError, "ncclCommGetAsyncError");
            RG_SYM(Send, "ncclSend");
            RG_SYM(Recv, "ncclRecv");
            RG_SYM(Bcast, "ncclBroadcast");
            RG_SYM(GroupStart, "ncclGroupStart");
            RG_SYM(GroupEnd, "ncclGroupEnd");
            RG_SYM(GetErrorString, "ncclGetErrorString");
#undef RG_SYM
            api.ok = api.GetUniqueId && api.CommInitRank && api.CommDestroy && api.Send && api.Recv &&
                     api.Bcast && api.GroupStart && api.GroupEnd && api.GetErrorString;
        }
    }
    if (!api.ok)
        return set_error(RODINIA_E_NCCL, "NCCL not loadable (set RODINIA_NCCL_LIB to libnccl.so.2)");
    *out = &api;
    return RODINIA_OK;
}

#define RG_NCCL(api, x)                                                                         \
    do {                                                                                        \
        ncclResult_t _r = (x);                                                                  \
        if (_r != ncclSuccess) return set_error(RODINIA_E_NCCL, "%s: %s", #x, (api)->GetErrorString(_r)); \
    } while (0)

// ------------------------------------------------------------------ slabs and plans (host only)
static void slab_of(int64_t R, int P, int r, int64_t* row0, int64_t* n) {
    const int64_t a = (int64_t)r * R / P, b = (int64_t)(r + 1) * R / P;
    *row0 = a;
    *n = b - a;
}

// The schedule of one rank (rodinia_dist_plan): halo depths, exchange period and sizes.
//  hotspot: D = steps per launch of the granularity; halos D / D; sends D / D rows.
//  srad:    D = exchange period; halos D above / 2D below; sends 2D rows up, D down; cone window.
static rodinia_status plan_of(rodinia_kernel k, int64_t R, int64_t C, int P, int r, int iters, int64_t r1,
                              int64_t r2, int64_t c1, int64_t c2, int D, rodinia_dist_plan* o) {
    memset(o, 0, sizeof *o);
    slab_of(R, P, r, &o->row0, &o->own);
    const int up = k == RODINIA_SRAD ? 2 * D : D;  // rows a slab sends to the rank above
    const int down = D;                           // rows a slab sends to the rank below
    o->period = D;
    o->top = r > 0 ? down : 0;
    o->bot = r + 1 < P ? up : 0;
    o->send_up = r > 0 ? up : 0;
    o->send_down = r + 1 < P ? down : 0;
    o->exchanges = P > 1 ? (iters + D - 1) / D : 0;
    int64_t own_min = R / P;  // smallest slab
    if (P > 1 && own_min < std::max(up, down))
        return set_error(RODINIA_E_ILLEGAL_FACTOR,
                         "dist: slabs of %lld rows are thinner than the halo depth %d; use fewer ranks or a "
                         "smaller temporal depth", (long long)own_min, std::max(up, down));
    // hotspot overlap: the owned rows determine output rows [D, own - D) by themselves
    o->overlap = (k == RODINIA_HOTSPOT && P > 1 && o->own > 2 * D) ? 1 : 0;
    if (k == RODINIA_SRAD) {
        o->cone_r0 = std::max<int64_t>(0, r1 - iters);
        o->cone_r1 = std::min<int64_t>(R, r2 + 2 * (int64_t)iters + 3);
        o->cone_c0 = std::max<int64_t>(0, c1 - iters);
        o->cone_c1 = std::min<int64_t>(C, c2 + 2 * (int64_t)iters + 3);
    }
    return RODINIA_OK;
}

static int srad_auto_depth(int64_t R, int P) {
    if (P == 1) return 1;
    const int64_t own_min = R / P;
    return (int)std::max<int64_t>(1, std::min<int64_t>(8, own_min / 2));
}

// Halo exchange of buffer `which` of every local slab: every slab sends its first `up` own
// rows to the slab above (its bottom halo, depth up) and its last `down` own rows to the slab
// below (its top halo, depth down).
static rodinia_status exchange(rodinia_comm* c, std::vector<Slab>& sl, int which, int C, int up, int down,
                               bool aux, cudaStream_t s) {
    const size_t rowb = (size_t)C * sizeof(float);
    auto base = [&](Slab& x) { return aux ? x.aux : x.buf[which]; };
    if (c->kind == 1) {
        for (size_t i = 0; i < sl.size(); ++i) {
            Slab& x = sl[i];
            if (i > 0) {
                Slab& a = sl[i - 1];  // my first `up` own rows -> a's bottom halo
                RG_CUDA(cudaMemcpyAsync(base(a) + (size_t)(a.top + a.own) * C, base(x) + (size_t)x.top * C,
                                        up * rowb, cudaMemcpyDeviceToDevice, s));
            }
            if (i + 1 < sl.size()) {
                Slab& b = sl[i + 1];  // my last `down` own rows -> b's top halo
                RG_CUDA(cudaMemcpyAsync(base(b), base(x) + (size_t)(x.top + x.own - down) * C, down * rowb,
                                        cudaMemcpyDeviceToDevice, s));
            }
        }
        return RODINIA_OK;
    }
    NcclApi* api;
    RG_TRY(nccl_api(&api));
    Slab& x = sl[0];
    const int r = c->rank, P = c->nranks;
    RG_NCCL(api, api->GroupStart());
    if (r > 0) {
        RG_NCCL(api, api->Send(base(x) + (size_t)x.top * C, (size_t)up * C, ncclFloat32, r - 1, c->nccl, s));
        RG_NCCL(api, api->Recv(base(x), (size_t)down * C, ncclFloat32, r - 1, c->nccl, s));
    }
    if (r + 1 < P) {
        RG_NCCL(api, api->Send(base(x) + (size_t)(x.top + x.own - down) * C, (size_t)down * C, ncclFloat32, r + 1,
                               c->nccl, s));
        RG_NCCL(api, api->Recv(base(x) + (size_t)(x.top + x.own) * C, (size_t)up * C, ncclFloat32, r + 1,
                               c->nccl, s));
    }
    RG_NCCL(api, api->GroupEnd());
    return RODINIA_OK;
}

static void free_slab(Slab& x) {
    for (float* p : {x.buf[0], x.buf[1], x.aux, x.scr, x.strip[0], x.strip[1], x.strip_scr})
        if (p) cudaFree(p);
    memset(&x, 0, sizeof x);
}

static rodinia_status dev_alloc(float** p, size_t floats) {
    if (cudaMalloc((void**)p, std::max<size_t>(floats, 1) * sizeof(float)) != cudaSuccess) {
        cudaGetLastError();
        *p = nullptr;
        return set_error(RODINIA_E_NOMEM, "dist: slab allocation of %zu floats failed", floats);
    }
    return RODINIA_OK;
}

// The slabs this process holds (NCCL: its own; LOCAL: all), with halo depths from the plan.
static rodinia_status make_slabs(rodinia_comm* c, rodinia_kernel k, int64_t R, int64_t C, int iters, int D,
                                 std::vector<Slab>* out) {
    const int P = c->nranks;
    std::vector<int> ranks;
    if (c->kind == 1)
        for (int r = 0; r < P; ++r) ranks.push_back(r);
    else
        ranks.push_back(c->rank);
    for (int r : ranks) {
        rodinia_dist_plan pl;
        RG_TRY(plan_of(k, R, C, P, r, iters, 0, 0, 0, 0, D, &pl));
        Slab x;
        memset(&x, 0, sizeof x);
        x.rank = r;
        x.row0 = pl.row0;
        x.own = (int)pl.own;
        x.top = pl.top;
        x.bot = pl.bot;
        out->push_back(x);
    }
    return RODINIA_OK;
}

static rodinia_status comm_setup(rodinia_comm* c) {
    int dev = 0;
    RG_CUDA(cudaGetDevice(&dev));
    if (c->side && c->dev == dev) return RODINIA_OK;
    RG_CUDA(cudaStreamCreateWithFlags(&c->side, cudaStreamNonBlocking));
    RG_CUDA(cudaEventCreateWithFlags(&c->ev_ready, cudaEventDisableTiming));
    RG_CUDA(cudaEventCreateWithFlags(&c->ev_strips, cudaEventDisableTiming));
    RG_CUDA(cudaEventCreateWithFlags(&c->ev_done, cudaEventDisableTiming));
    c->dev = dev;
    c->done_recorded = false;
    return RODINIA_OK;
}

// pointer of local slab i among the caller's arguments (NCCL: the pointer itself; LOCAL: array)
static const float* arg_ptr(rodinia_comm* c, const void* a, size_t i) {
    return c->kind == 1 ? ((const float* const*)a)[i] : (const float*)a;
}

}  // namespace rg

using namespace rg;

// ===================================================================== exported: comm
extern "C" rodinia_status rodinia_slab(int64_t R, int32_t P, int32_t r, int64_t* row0, int64_t* nrows) {
    if (R < 1 || P < 1 || r < 0 || r >= P || !row0 || !nrows) return set_error(RODINIA_E_INVALID, "slab: bad arguments");
    slab_of(R, P, r, row0, nrows);
    return RODINIA_OK;
}

static rodinia_status resolve_hotspot(int64_t R, int64_t C, int iters, int P, const rodinia_granularity* g,
                                      rodinia_granularity* gg, const hotspot::DirectVariant** dv,
                                      const hotspot::StreamVariant** sv) {
    int64_t row0, own0;
    slab_of(R, P, 0, &row0, &own0);
    if (!gran_is_zero(g)) *gg = *g;
    else {
        rodinia_problem pb{own0, C, iters, P};
        if (!tune_cache_lookup(RODINIA_HOTSPOT, pb, gg)) *gg = default_gran(RODINIA_HOTSPOT, pb);
    }
    // the largest buffer a launch sees: the biggest slab with both halos
    const int h = (gg->flags & RODINIA_STREAM) ? std::max(1, gg->temporal) : 1;
    return hotspot::check(*gg, (R + P - 1) / P + 2 * h, C, dv, sv);
}

static rodinia_status resolve_srad(int64_t R, int64_t C, int niter, int P, const rodinia_granularity* g,
                                   rodinia_granularity* gg, int* D) {
    int64_t row0, own0;
    slab_of(R, P, 0, &row0, &own0);
    if (!gran_is_zero(g)) {
        *gg = *g;
        *D = std::max(1, g->temporal);  // exchange period / halo depth
    } else {
        rodinia_problem pb{own0, C, niter, P};
        if (!tune_cache_lookup(RODINIA_SRAD, pb, gg)) *gg = default_gran(RODINIA_SRAD, pb);
        *D = srad_auto_depth(R, P);
    }
    gg->temporal = 1;  // every srad launch is one iteration; D only sets the exchange period
    return RODINIA_OK;
}

extern "C" rodinia_status rodinia_dist_schedule(rodinia_kernel k, int64_t R, int64_t C, int32_t P, int32_t r,
                                            int32_t iters, int64_t r1, int64_t r2, int64_t c1, int64_t c2,
                                            const rodinia_granularity* g, rodinia_dist_plan* out) {
    if (!out || R < 1 || C < 1 || P < 1 || r < 0 || r >= P || iters < 0 || R < P)
        return set_error(RODINIA_E_INVALID, "dist_schedule: bad arguments");
    if (k == RODINIA_HOTSPOT) {
        rodinia_granularity gg;
        const hotspot::DirectVariant* dv;
        const hotspot::StreamVariant* sv;
        RG_TRY(resolve_hotspot(R, C, iters, P, g, &gg, &dv, &sv));
        return plan_of(k, R, C, P, r, iters, 0, 0, 0, 0, hotspot::temporal_of(sv), out);
    }
    if (k == RODINIA_SRAD) {
        if (r1 < 0 || c1 < 0 || r2 < r1 || c2 < c1 || r2 >= R || c2 >= C)
            return set_error(RODINIA_E_INVALID, "dist_schedule: ROI outside the grid");
        rodinia_granularity gg;
        int D;
        RG_TRY(resolve_srad(R, C, iters, P, g, &gg, &D));
        return plan_of(k, R, C, P, r, iters, r1, r2, c1, c2, D, out);
    }
    return set_error(RODINIA_E_INVALID, "dist_schedule: only hotspot and srad are sharded (pathfinder and lud run "
                                        "as replicas, DESIGN.md §6)");
}

extern "C" rodinia_status rodinia_comm_unique_id(uint8_t id[128]) {
    if (!id) return set_error(RODINIA_E_INVALID, "comm_unique_id: null");
    NcclApi* api;
    RG_TRY(nccl_api(&api));
    ncclUniqueId u;
    RG_NCCL(api, api->GetUniqueId(&u));
    static_assert(sizeof(u) == 128, "ncclUniqueId size");
    memcpy(id, &u, 128);
    return RODINIA_OK;
}

extern "C" rodinia_status rodinia_comm_init(rodinia_comm** out, int32_t nranks, int32_t rank, const uint8_t id[128]) {
    if (!out || !id || nranks < 1 || rank < 0 || rank >= nranks) return set_error(RODINIA_E_INVALID, "comm_init: bad arguments");
    DeviceInfo di;
    RG_TRY(device_info(&di));
    NcclApi* api;
    RG_TRY(nccl_api(&api));
    ncclUniqueId u;
    memcpy(&u, id, 128);
    rodinia_comm* c = new rodinia_comm();
    c->kind = 0;
    c->nranks = nranks;
    c->rank = rank;
    ncclResult_t r = api->CommInitRank(&c->nccl, nranks, u, rank);
    if (r != ncclSuccess) {
        delete c;
        return set_error(RODINIA_E_NCCL, "ncclCommInitRank: %s", api->GetErrorString(r));
    }
    *out = c;
    return RODINIA_OK;
}

extern "C" rodinia_status rodinia_comm_init_local(rodinia_comm** out, int32_t nranks) {
    if (!out || nranks < 1 || nranks > 1024) return set_error(RODINIA_E_INVALID, "comm_init_local: bad arguments");
    rodinia_comm* c = new rodinia_comm();
    c->kind = 1;
    c->nranks = nranks;
    c->rank = 0;
    c->nccl = nullptr;
    *out = c;
    return RODINIA_OK;
}

static void release_hs(rodinia_comm* c) {
    for (auto& x : c->hs.sl) free_slab(x);
    c->hs.sl.clear();
    c->hs.R = c->hs.C = 0;
}

static void release_sr(rodinia_comm* c) {
    for (auto& x : c->sr.sl) {
        x.buf[1] = nullptr;  // the engine's ping-pong buffer (freed with the engine)
        free_slab(x);
    }
    for (auto& e : c->sr.eng) srad::engine_free(&e, nullptr);
    if (c->sr.have_we) srad::engine_free(&c->sr.we, nullptr);
    if (c->sr.W) cudaFree(c->sr.W);
    c->sr.sl.clear();
    c->sr.eng.clear();
    c->sr.W = nullptr;
    c->sr.have_we = false;
    c->sr.R = c->sr.C = 0;
}

extern "C" rodinia_status rodinia_comm_destroy(rodinia_comm* c) {
    if (!c) return set_error(RODINIA_E_INVALID, "comm_destroy: null");
    {
        std::lock_guard<std::mutex> lk(c->mu);
        if (c->side) {
            cudaDeviceSynchronize();  // buffers may still be in use by enqueued work
            release_hs(c);
            release_sr(c);
            cudaStreamDestroy(c->side);
            cudaEventDestroy(c->ev_ready);
            cudaEventDestroy(c->ev_strips);
            cudaEventDestroy(c->ev_done);
            for (auto e : c->ev_cone) cudaEventDestroy(e);
            c->ev_cone.clear();
            cudaGetLastError();  // teardown errors are not reported to later calls
        }
        if (c->kind == 0 && c->nccl) {
            NcclApi* api;
            if (nccl_api(&api) == RODINIA_OK) api->CommDestroy(c->nccl);
        }
    }
    delete c;
    return RODINIA_OK;
}

// ===================================================================== exported: hotspot_dist
// One full period with overlap: side stream = exchange + boundary strips into
// strip buffers, compute stream = interior launch on the owned rows, then the strips' valid
// rows are copied into the output buffer.
static rodinia_status hs_period_overlap(rodinia_comm* c, std::vector<Slab>& sl, int cur, int C, int D,
                                        const HsCoef& cf, const rodinia_granularity& gg,
                                        const hotspot::DirectVariant* dv, const hotspot::StreamVariant* sv,
                                        cudaStream_t s) {
    const size_t rowb = (size_t)C * sizeof(float);
    RG_CUDA(cudaEventRecord(c->ev_ready, s));
    RG_CUDA(cudaStreamWaitEvent(c->side, c->ev_ready, 0));
    RG_TRY(exchange(c, sl, cur, C, D, D, false, c->side));
    for (auto& x : sl) {
        // top strip: buffer rows [0, top + 2D) -> outputs [top, top + D)
        const int tr = x.top + 2 * D;
        RG_TRY(hotspot::run(x.buf[cur], x.aux, x.strip[0], x.strip_scr, tr, C, D, cf, gg, dv, sv, c->side));
        // bottom strip: buffer rows [top + own - 2D, rows) -> outputs [D, 2D) of the strip
        const int b0 = x.top + x.own - 2 * D, br = 2 * D + x.bot;
        RG_TRY(hotspot::run(x.buf[cur] + (size_t)b0 * C, x.aux + (size_t)b0 * C, x.strip[1], x.strip_scr, br, C, D,
                            cf, gg, dv, sv, c->side));
    }
    RG_CUDA(cudaEventRecord(c->ev_strips, c->side));
    for (auto& x : sl)  // interior: the owned rows alone, outputs [D, own - D) valid
        RG_TRY(hotspot::run(x.buf[cur] + (size_t)x.top * C, x.aux + (size_t)x.top * C,
                            x.buf[1 - cur] + (size_t)x.top * C, x.scr, x.own, C, D, cf, gg, dv, sv, s));
    RG_CUDA(cudaStreamWaitEvent(s, c->ev_strips, 0));
    for (auto& x : sl) {
        RG_CUDA(cudaMemcpyAsync(x.buf[1 - cur] + (size_t)x.top * C, x.strip[0] + (size_t)x.top * C, D * rowb,
                                cudaMemcpyDeviceToDevice, s));
        RG_CUDA(cudaMemcpyAsync(x.buf[1 - cur] + (size_t)(x.top + x.own - D) * C, x.strip[1] + (size_t)D * C,
                                D * rowb, cudaMemcpyDeviceToDevice, s));
    }
    return RODINIA_OK;
}

extern "C" rodinia_status rodinia_hotspot_dist(rodinia_comm* c, const void* temp_local, const void* power_local,
                                               void* out_local, int64_t R, int64_t C, int32_t iters,
                                               const rodinia_hotspot_coeffs* coeffs, const rodinia_granularity* g,
                                               void* stream) {
    if (!c || !temp_local || !power_local || !out_local) return set_error(RODINIA_E_INVALID, "hotspot_dist: null argument");
    if (R < 1 || C < 1 || iters < 0 || R < c->nranks) return set_error(RODINIA_E_INVALID, "hotspot_dist: bad sizes");
    if (R > (1ll << 31) - 1 || C > (1ll << 31) - 1) return set_error(RODINIA_E_INVALID, "hotspot_dist: grid too large");
    if (c->kind == 1)
        for (int i = 0; i < c->nranks; ++i)
            if (!arg_ptr(c, temp_local, i) || !arg_ptr(c, power_local, i) || !((float* const*)out_local)[i])
                return set_error(RODINIA_E_INVALID, "hotspot_dist: null slab pointer");
    rodinia_granularity gg;
    const hotspot::DirectVariant* dv;
    const hotspot::StreamVariant* sv;
    RG_TRY(resolve_hotspot(R, C, iters, c->nranks, g, &gg, &dv, &sv));
    const int D = hotspot::temporal_of(sv);
    rodinia_hotspot_coeffs cc;
    if (coeffs) cc = *coeffs;
    else rodinia_hotspot_coeffs_rodinia(R, C, 0.016, 0.016, &cc);
    const HsCoef cf = hs_derive(cc.k, cc.rx, cc.ry, cc.rz);  // state form (hs_cell.cuh)
    std::vector<Slab> want;
    RG_TRY(make_slabs(c, RODINIA_HOTSPOT, R, C, iters, D, &want));
    DeviceInfo di;
    RG_TRY(device_info(&di));
    std::lock_guard<std::mutex> lk(c->mu);
    RG_TRY(comm_setup(c));
    cudaStream_t s = (cudaStream_t)stream;
    // the communicator's buffers are reused: order this call after the previous one
    if (c->done_recorded) RG_CUDA(cudaStreamWaitEvent(s, c->ev_done, 0));
    // persistent slab buffers (reallocated only when the shape or halo depth changes)
    auto& hc = c->hs;
    if (hc.R != R || hc.C != C || hc.D != D || hc.sl.size() != want.size()) {
        RG_CUDA(cudaStreamSynchronize(s));
        release_hs(c);
        for (auto& x : want) {
            const size_t n = (size_t)x.rows() * C, ns = (size_t)(x.top + 2 * D + std::max(x.bot, D)) * C;
            RG_TRY(dev_alloc(&x.buf[0], n));
            RG_TRY(dev_alloc(&x.buf[1], n));
            RG_TRY(dev_alloc(&x.aux, n));
            RG_TRY(dev_alloc(&x.scr, n));
            RG_TRY(dev_alloc(&x.strip[0], ns));
            RG_TRY(dev_alloc(&x.strip[1], ns));
            RG_TRY(dev_alloc(&x.strip_scr, ns));
            hc.sl.push_back(x);
        }
        hc.R = R;
        hc.C = C;
        hc.D = D;
    }
    std::vector<Slab>& sl = hc.sl;
    const size_t rowb = (size_t)C * sizeof(float);
    for (size_t i = 0; i < sl.size(); ++i) {
        Slab& x = sl[i];
        // T -> u = T - amb and P -> kP = k*P straight into the owned rows (halos arrive converted)
        hotspot::convert(arg_ptr(c, temp_local, i), x.buf[0] + (size_t)x.top * C, (int64_t)x.own * C, 0, cc.amb, s);
        hotspot::convert(arg_ptr(c, power_local, i), x.aux + (size_t)x.top * C, (int64_t)x.own * C, 1, cc.k, s);
    }
    rodinia_status st = RODINIA_OK;
    if (c->nranks > 1) st = exchange(c, sl, 0, (int)C, D, D, true, s);
    bool overlap = c->nranks > 1;
    for (auto& x : sl) overlap = overlap && x.own > 2 * D;
    int cur = 0;
    for (int done = 0; st == RODINIA_OK && done < iters;) {
        const int steps = std::min(D, iters - done);
        if (overlap && steps == D && hotspot::num_launches(D, sv) == 1) {
            st = hs_period_overlap(c, sl, cur, (int)C, D, cf, gg, dv, sv, s);
        } else {
            if (c->nranks > 1) st = exchange(c, sl, cur, (int)C, D, D, false, s);
            for (size_t i = 0; i < sl.size() && st == RODINIA_OK; ++i) {
                Slab& x = sl[i];
                st = hotspot::run(x.buf[cur], x.aux, x.buf[1 - cur], x.scr, x.rows(), (int)C, steps, cf, gg, dv, sv, s);
            }
        }
        cur = 1 - cur;
        done += steps;
    }
    for (size_t i = 0; i < sl.size() && st == RODINIA_OK; ++i) {
        Slab& x = sl[i];
        float* dst = c->kind == 1 ? ((float* const*)out_local)[i] : (float*)out_local;
        hotspot::convert(x.buf[cur] + (size_t)x.top * C, dst, (int64_t)x.own * C, 2, cc.amb, s);  // u -> T
    }
    (void)rowb;
    if (cudaEventRecord(c->ev_done, s) == cudaSuccess) c->done_recorded = true;
    if (st == RODINIA_OK) {
        const cudaError_t ce = cudaGetLastError();
        if (ce != cudaSuccess) st = cuda_error(ce, "hotspot_dist", __FILE__, __LINE__);
    }
    return st;
}

// ===================================================================== exported: srad_dist
extern "C" rodinia_status rodinia_srad_dist(rodinia_comm* c, void* J_local, int64_t R, int64_t C, int64_t r1,
                                            int64_t r2, int64_t c1, int64_t c2, float lambda, int32_t niter,
                                            const rodinia_granularity* g, void* stream) {
    if (!c || !J_local) return set_error(RODINIA_E_INVALID, "srad_dist: null argument");
    if (R < 1 || C < 1 || niter < 0 || R < c->nranks) return set_error(RODINIA_E_INVALID, "srad_dist: bad sizes");
    if (R > (1ll << 31) - 1 || C > (1ll << 31) - 1) return set_error(RODINIA_E_INVALID, "srad_dist: grid too large");
    if (r1 < 0 || c1 < 0 || r2 < r1 || c2 < c1 || r2 >= R || c2 >= C)
        return set_error(RODINIA_E_INVALID, "srad_dist: ROI outside the grid");
    if (!std::isfinite(lambda)) return set_error(RODINIA_E_INVALID, "srad_dist: lambda not finite");
    if (c->kind == 1)
        for (int i = 0; i < c->nranks; ++i)
            if (!((float* const*)J_local)[i]) return set_error(RODINIA_E_INVALID, "srad_dist: null slab pointer");
    rodinia_granularity gg;
    int D;
    RG_TRY(resolve_srad(R, C, niter, c->nranks, g, &gg, &D));
    srad::Plan p;
    RG_TRY(srad::plan(gg, &p));
    std::vector<Slab> want;
    RG_TRY(make_slabs(c, RODINIA_SRAD, R, C, niter, D, &want));
    DeviceInfo di;
    RG_TRY(device_info(&di));
    RG_TRY(srad::take_sticky());
    if (niter == 0) return RODINIA_OK;
    if (p.v && p.smem > 48 * 1024)
        RG_CUDA(cudaFuncSetAttribute((const void*)p.v->fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p.smem));
    std::lock_guard<std::mutex> lk(c->mu);
    RG_TRY(comm_setup(c));
    cudaStream_t s = (cudaStream_t)stream;
    const size_t rowb = (size_t)C * sizeof(float);
    if (c->done_recorded) RG_CUDA(cudaStreamWaitEvent(s, c->ev_done, 0));  // buffers are reused

    // ---- the ROI's dependency-cone window (plan_of: rows [r1-n, r2+2n+3) x cols likewise)
    rodinia_dist_plan pl0;
    RG_TRY(plan_of(RODINIA_SRAD, R, C, c->nranks, 0, niter, r1, r2, c1, c2, D, &pl0));
    const int64_t wr0 = pl0.cone_r0, wr1 = pl0.cone_r1, wc0 = pl0.cone_c0, wc1 = pl0.cone_c1;
    const int WR = (int)(wr1 - wr0), WC = (int)(wc1 - wc0);

    // ---- persistent slabs, engines and window (reallocated when the shape / plan changes)
    auto& sc = c->sr;
    const bool same = sc.R == R && sc.C == C && sc.D == D && sc.niter_cap >= niter && sc.WR == WR && sc.WC == WC &&
                      !memcmp(&sc.g, &gg, sizeof gg) && sc.sl.size() == want.size();
    if (!same) {
        RG_CUDA(cudaStreamSynchronize(s));
        release_sr(c);
        for (auto& x : want) {
            RG_TRY(dev_alloc(&x.buf[0], (size_t)x.rows() * C));
            sc.sl.push_back(x);
        }
        sc.eng.resize(want.size());
        RG_TRY(dev_alloc(&sc.W, (size_t)WR * WC));
        RG_TRY(srad::engine_alloc(&sc.we, p, WR, WC, niter, s));
        sc.have_we = true;
        for (size_t i = 0; i < want.size(); ++i) {
            RG_TRY(srad::engine_alloc(&sc.eng[i], p, sc.sl[i].rows(), (int)C, niter, s));
            sc.sl[i].buf[1] = sc.eng[i].jb;
            sc.eng[i].its = sc.we.its;  // q0sqr(t) read from the cone engine's table (no copy)
        }
        sc.R = R; sc.C = C; sc.D = D; sc.niter_cap = niter; sc.WR = WR; sc.WC = WC; sc.g = gg;
    }
    std::vector<Slab>& sl = sc.sl;
    rodinia_status st = RODINIA_OK;

    // ---- q0sqr(t) from the ROI's dependency cone (no per-iteration collective)
    float* W = sc.W;
    NcclApi* api = nullptr;
    if (c->kind == 0 && c->nranks > 1) st = nccl_api(&api);
    if (st == RODINIA_OK && api) {
        ncclResult_t r = api->GroupStart();
        for (int q = 0; q < c->nranks && r == ncclSuccess; ++q) {
            int64_t q0, qn;
            slab_of(R, c->nranks, q, &q0, &qn);
            const int64_t a = std::max(q0, wr0), b = std::min(q0 + qn, wr1);
            if (a >= b) continue;
            float* part = W + (size_t)(a - wr0) * WC;
            if (q == c->rank)  // owner packs its rows of the window
                cudaMemcpy2DAsync(part, WC * sizeof(float), (const float*)J_local + (size_t)(a - q0) * C + wc0,
                                  rowb, WC * sizeof(float), (size_t)(b - a), cudaMemcpyDeviceToDevice, s);
            r = api->Bcast(part, part, (size_t)(b - a) * WC, ncclFloat32, q, c->nccl, s);
        }
        ncclResult_t r2e = api->GroupEnd();
        if (r != ncclSuccess || r2e != ncclSuccess)
            st = set_error(RODINIA_E_NCCL, "srad_dist: cone broadcast failed");
    } else if (st == RODINIA_OK) {
        for (size_t i = 0; i < sl.size(); ++i) {
            const int64_t q0 = sl[i].row0, qn = sl[i].own;
            const int64_t a = std::max(q0, wr0), b = std::min(q0 + qn, wr1);
            if (a >= b) continue;
            const float* src = (c->kind == 1 ? ((float* const*)J_local)[i] : (float*)J_local);
            cudaMemcpy2DAsync(W + (size_t)(a - wr0) * WC, WC * sizeof(float), src + (size_t)(a - q0) * C + wc0,
                              rowb, WC * sizeof(float), (size_t)(b - a), cudaMemcpyDeviceToDevice, s);
        }
    }
    // The cone's iterations (one statistics + one update launch each on a window of at most
    // (3n)^2 cells: launch-latency bound) run on the side stream, one exchange period ahead of
    // the slab iterations, which wait for period p's q0sqr values only (ev_cone[p]).  NCCL work
    // stays on the compute stream.
    const int nper = (niter + D - 1) / D;
    while ((int)c->ev_cone.size() < nper) {
        cudaEvent_t e;
        RG_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        c->ev_cone.push_back(e);
    }
    if (st == RODINIA_OK) {
        RG_CUDA(cudaEventRecord(c->ev_ready, s));  // the window's J0 has been gathered
        RG_CUDA(cudaStreamWaitEvent(c->side, c->ev_ready, 0));
        float* wc = W;
        float* wo = sc.we.jb;
        for (int q = 0; q < nper; ++q) {
            float* res = srad::engine_steps(&sc.we, wc, wo, q * D, std::min(niter, (q + 1) * D), true,
                                            (int)(r1 - wr0), (int)(c1 - wc0), (int)(r2 - r1 + 1), (int)(c2 - c1 + 1),
                                            0.25f * lambda, c->side);
            wo = (res == wc) ? wo : wc;
            wc = res;
            RG_CUDA(cudaEventRecord(c->ev_cone[q], c->side));
        }
    }

    // ---- slabs: halo D above, 2D below, exchange every D iterations
    for (size_t i = 0; i < sl.size() && st == RODINIA_OK; ++i) {
        Slab& x = sl[i];
        const float* src = (c->kind == 1 ? ((float* const*)J_local)[i] : (float*)J_local);
        if (cudaMemcpyAsync(x.buf[0] + (size_t)x.top * C, src, x.own * rowb, cudaMemcpyDeviceToDevice, s) != cudaSuccess)
            st = cuda_error(cudaGetLastError(), "srad_dist copy-in", __FILE__, __LINE__);
    }
    std::vector<float*> cur(sl.size()), oth(sl.size());
    for (size_t i = 0; i < sl.size(); ++i) { cur[i] = sl[i].buf[0]; oth[i] = sl[i].buf[1]; }
    for (int it = 0, q = 0; st == RODINIA_OK && it < niter; it += D, ++q) {
        if (c->nranks > 1) {
            // exchange on whichever buffer currently holds J (same parity on every slab)
            const int which = (cur[0] == sl[0].buf[0]) ? 0 : 1;
            st = exchange(c, sl, which, (int)C, 2 * D, D, false, s);
        }
        if (st == RODINIA_OK && cudaStreamWaitEvent(s, c->ev_cone[q], 0) != cudaSuccess)
            st = cuda_error(cudaGetLastError(), "srad_dist cone wait", __FILE__, __LINE__);
        for (size_t i = 0; i < sl.size() && st == RODINIA_OK; ++i) {
            float* res = srad::engine_steps(&sc.eng[i], cur[i], oth[i], it, std::min(niter, it + D), false, 0, 0, 1, 1,
                                            0.25f * lambda, s);
            oth[i] = (res == cur[i]) ? oth[i] : cur[i];
            cur[i] = res;
        }
    }
    for (size_t i = 0; i < sl.size() && st == RODINIA_OK; ++i) {
        Slab& x = sl[i];
        float* dst = c->kind == 1 ? ((float* const*)J_local)[i] : (float*)J_local;
        if (cudaMemcpyAsync(dst, cur[i] + (size_t)x.top * C, x.own * rowb, cudaMemcpyDeviceToDevice, s) != cudaSuccess)
            st = cuda_error(cudaGetLastError(), "srad_dist copy-out", __FILE__, __LINE__);
    }
    if (cudaEventRecord(c->ev_done, s) == cudaSuccess) c->done_recorded = true;
    if (st == RODINIA_OK) {
        const cudaError_t ce = cudaGetLastError();
        if (ce != cudaSuccess) st = cuda_error(ce, "srad_dist", __FILE__, __LINE__);
    }
    return st;
}

// ===================================================================== 2-D block-cyclic LU
// SURVEY §8(f) #3 ("then a 2-D block-cyclic multi-GPU LU"), DESIGN.md §6.  Process grid
// prow x pcol (rank r = pr * pcol + pc), NB = 128 blocks; global block (I, J) lives on rank
// (I mod prow, J mod pcol).  Local matrix: the rank's block rows in increasing I, its block
// columns in increasing J, row-major, leading dimension = local columns (rodinia_lud_dist_layout).
// Right-looking, per block column k (owner (pk, qk) = (k mod prow, k mod pcol)):
//   1. (pk, qk) factors A_kk (ldist::diag) and broadcasts its images to every rank;
//   2. process column qk solves its L_Ik, process row pk its U_kJ (ldist::trsm), each writing
//      the hi/lo operand image of its panel;
//   3. L images travel along process rows, U images along process columns (send/recv);
//   4. every rank updates its trailing blocks (ldist::update, tensor cores): first the blocks of
//      block row / column k+1 (the next step's panel, on the main stream), then the rest on a
//      low-priority side stream, which runs under the next step's 1.-3. (look-ahead; the images
//      are double-buffered by step parity, and the next step's updates wait for the rest).
namespace rg {
static int64_t bc_extent(int64_t n, int P, int p) {  // rows of the global blocks I = p (mod P)
    const int64_t nb = (n + ldist::NB - 1) / ldist::NB;
    int64_t e = 0;
    for (int64_t I = p; I < nb; I += P) e += std::min<int64_t>(ldist::NB, n - I * ldist::NB);
    return e;
}
static int64_t bc_blocks_le(int64_t k, int P, int p) {  // local blocks I = p (mod P) with I <= k
    return k < p ? 0 : (k - p) / P + 1;
}
struct LudRank {
    int r, pr, pc;
    float* A;
    int64_t mloc, nloc;
    float** slot;
    float* mimg;
    float* ia[2];
    float* ib[2];
};
}  // namespace rg

extern "C" rodinia_status rodinia_lud_dist_layout(int64_t n, int32_t prow, int32_t pcol, int32_t rank,
                                                  int64_t* mloc, int64_t* nloc) {
    if (n < 1 || prow < 1 || pcol < 1 || rank < 0 || rank >= prow * pcol || !mloc || !nloc)
        return set_error(RODINIA_E_INVALID, "lud_dist_layout: bad arguments");
    *mloc = bc_extent(n, prow, rank / pcol);
    *nloc = bc_extent(n, pcol, rank % pcol);
    return RODINIA_OK;
}

extern "C" rodinia_status rodinia_lud_dist(rodinia_comm* c, void* a_local, int64_t n, int32_t prow, int32_t pcol,
                                           void* stream) {
    if (!c || !a_local || n < 1 || prow < 1 || pcol < 1)
        return set_error(RODINIA_E_INVALID, "lud_dist: bad arguments");
    if (prow * pcol != c->nranks)
        return set_error(RODINIA_E_INVALID, "lud_dist: process grid %d x %d != %d ranks", prow, pcol, c->nranks);
    if (n > (int64_t)1 << 20) return set_error(RODINIA_E_INVALID, "lud_dist: n too large");
    std::lock_guard<std::mutex> lk(c->mu);
    cudaStream_t us = (cudaStream_t)stream;
    const int P = c->nranks;
    std::vector<LudRank> rk;
    for (int r = 0; r < P; ++r) {
        if (c->kind != 1 && r != c->rank) continue;
        LudRank x;
        memset(&x, 0, sizeof x);
        x.r = r;
        x.pr = r / pcol;
        x.pc = r % pcol;
        x.A = (float*)arg_ptr(c, a_local, rk.size());
        x.mloc = bc_extent(n, prow, x.pr);
        x.nloc = bc_extent(n, pcol, x.pc);
        if (x.mloc > 0 && x.nloc > 0 && !x.A) return set_error(RODINIA_E_INVALID, "lud_dist: null local matrix");
        rk.push_back(x);
    }
    // streams: the main chain on a high-priority stream, the remainder updates on a low-priority
    // side stream; both are joined to the caller's stream at entry and exit
    int prio_lo = 0, prio_hi = 0;
    cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
    cudaStream_t s = nullptr, s2 = nullptr;
    cudaEvent_t ev_in = nullptr, ev_img = nullptr, ev_rest = nullptr;
    RG_CUDA(cudaStreamCreateWithPriority(&s, cudaStreamNonBlocking, prio_hi));
    RG_CUDA(cudaStreamCreateWithPriority(&s2, cudaStreamNonBlocking, prio_lo));
    RG_CUDA(cudaEventCreateWithFlags(&ev_in, cudaEventDisableTiming));
    RG_CUDA(cudaEventCreateWithFlags(&ev_img, cudaEventDisableTiming));
    RG_CUDA(cudaEventCreateWithFlags(&ev_rest, cudaEventDisableTiming));
    RG_CUDA(cudaEventRecord(ev_in, us));
    RG_CUDA(cudaStreamWaitEvent(s, ev_in, 0));
    RG_CUDA(cudaStreamWaitEvent(s2, ev_in, 0));
    auto cleanup = [&]() {
        cudaEventRecord(ev_rest, s2);  // join the side stream, release the scratch, join the caller
        cudaStreamWaitEvent(s, ev_rest, 0);
        for (auto& x : rk)
            for (void* p : {(void*)x.slot, (void*)x.mimg, (void*)x.ia[0], (void*)x.ia[1], (void*)x.ib[0],
                            (void*)x.ib[1]})
                if (p) cudaFreeAsync(p, s);
        cudaEventRecord(ev_in, s);
        cudaStreamWaitEvent(us, ev_in, 0);
        cudaStreamDestroy(s);
        cudaStreamDestroy(s2);
        cudaEventDestroy(ev_in);
        cudaEventDestroy(ev_img);
        cudaEventDestroy(ev_rest);
    };
    bool alloc_ok = true;
    for (auto& x : rk) {
        const size_t fa = ldist::img_floats(std::max<int64_t>(x.mloc, 1));
        const size_t fb = ldist::img_floats(std::max<int64_t>(x.nloc, 1));
        alloc_ok = alloc_ok && cudaMallocAsync((void**)&x.slot, sizeof(float*), s) == cudaSuccess &&
                   cudaMallocAsync((void**)&x.mimg, ldist::mimg_floats() * sizeof(float), s) == cudaSuccess;
        for (int b = 0; b < 2; ++b)
            alloc_ok = alloc_ok && cudaMallocAsync((void**)&x.ia[b], fa * sizeof(float), s) == cudaSuccess &&
                       cudaMallocAsync((void**)&x.ib[b], fb * sizeof(float), s) == cudaSuccess;
        if (!alloc_ok) break;
    }
    if (!alloc_ok) {
        cudaGetLastError();
        cleanup();
        return set_error(RODINIA_E_NOMEM, "lud_dist: scratch allocation failed");
    }
    rodinia_status st = RODINIA_OK;
    for (auto& x : rk) {
        st = ldist::set_slot(x.slot, x.A, s);
        if (st != RODINIA_OK) { cleanup(); return st; }
    }
    NcclApi* api = nullptr;
    if (c->kind != 1 && P > 1) {
        st = nccl_api(&api);
        if (st != RODINIA_OK) { cleanup(); return st; }
    }
    const int64_t NB = ldist::NB, nb = (n + NB - 1) / NB;
    bool rest_pending = false;
    auto find = [&](int r) -> LudRank* {
        for (auto& x : rk)
            if (x.r == r) return &x;
        return nullptr;
    };
#define LD_TRY(x)                        \
    do {                                 \
        st = (x);                        \
        if (st != RODINIA_OK) goto done; \
    } while (0)
#define LD_CUDA(x, what)                                                                     \
    do {                                                                                     \
        cudaError_t _e = (x);                                                                \
        if (_e != cudaSuccess) { st = cuda_error(_e, what, __FILE__, __LINE__); goto done; } \
    } while (0)
    for (int64_t k = 0; k < nb; ++k) {
        const int pk = (int)(k % prow), qk = (int)(k % pcol), root = pk * pcol + qk;
        const int bk = (int)std::min<int64_t>(NB, n - k * NB);
        const int64_t lrk = (k / prow) * NB, lck = (k / pcol) * NB;  // block (k, k) on its owner
        const int par = (int)(k & 1);
        if (LudRank* o = find(root)) LD_TRY(ldist::diag(o->slot, (size_t)(lrk * o->nloc + lck), (int)o->nloc, bk, o->mimg, s, prio_hi));
        if (k == nb - 1) break;
        // 1. the diagonal block's images to every rank
        if (P > 1) {
            const size_t cnt = ldist::mimg_floats();
            if (c->kind == 1) {
                LudRank* o = find(root);
                for (auto& x : rk)
                    if (x.r != root)
                        LD_CUDA(cudaMemcpyAsync(x.mimg, o->mimg, cnt * sizeof(float), cudaMemcpyDeviceToDevice, s),
                                "lud_dist bcast");
            } else {
                ncclResult_t e = api->Bcast(rk[0].mimg, rk[0].mimg, cnt, ncclFloat32, root, c->nccl, s);
                if (e != ncclSuccess) { st = set_error(RODINIA_E_NCCL, "lud_dist bcast: %s", api->GetErrorString(e)); goto done; }
            }
        }
        // 2. panel solves into this step's images (the side stream's remainder update of step
        //    k-2 read them; the main stream waited for it before step k-1's updates)
        for (auto& x : rk) {
            const int64_t lr0 = bc_blocks_le(k, prow, x.pr) * NB, lc0 = bc_blocks_le(k, pcol, x.pc) * NB;
            ldist::TrsmJob jobs[2];
            int nj = 0;
            if (x.pc == qk && x.mloc > lr0)
                jobs[nj++] = ldist::TrsmJob{x.slot, (size_t)(lr0 * x.nloc + lck), (int)x.nloc, 1, (int)(x.mloc - lr0), x.ia[par],
                                            ldist::img_groups(x.mloc - lr0)};
            if (x.pr == pk && x.nloc > lc0)
                jobs[nj++] = ldist::TrsmJob{x.slot, (size_t)(lrk * x.nloc + lc0), (int)x.nloc, 0, (int)(x.nloc - lc0), x.ib[par],
                                            ldist::img_groups(x.nloc - lc0)};
            LD_TRY(ldist::trsm(jobs, nj, x.mimg, s, prio_hi));
        }
        // 3. L images along process rows (from (pr, qk)), U images along process columns (from (pk, pc))
        if (P > 1) {
            if (c->kind == 1) {
                for (auto& x : rk) {
                    const int64_t rows = x.mloc - bc_blocks_le(k, prow, x.pr) * NB;
                    const int64_t cols = x.nloc - bc_blocks_le(k, pcol, x.pc) * NB;
                    if (x.pc != qk && rows > 0)
                        LD_CUDA(cudaMemcpyAsync(x.ia[par], find(x.pr * pcol + qk)->ia[par],
                                                ldist::img_floats(rows) * sizeof(float), cudaMemcpyDeviceToDevice, s),
                                "lud_dist L image");
                    if (x.pr != pk && cols > 0)
                        LD_CUDA(cudaMemcpyAsync(x.ib[par], find(pk * pcol + x.pc)->ib[par],
                                                ldist::img_floats(cols) * sizeof(float), cudaMemcpyDeviceToDevice, s),
                                "lud_dist U image");
                }
            } else {
                LudRank& x = rk[0];
                const int64_t rows = x.mloc - bc_blocks_le(k, prow, x.pr) * NB;
                const int64_t cols = x.nloc - bc_blocks_le(k, pcol, x.pc) * NB;
                ncclResult_t e = api->GroupStart();
                if (rows > 0 && pcol > 1) {
                    const size_t cnt = ldist::img_floats(rows);
                    if (x.pc == qk) {
                        for (int q = 0; q < pcol && e == ncclSuccess; ++q)
                            if (q != qk) e = api->Send(x.ia[par], cnt, ncclFloat32, x.pr * pcol + q, c->nccl, s);
                    } else if (e == ncclSuccess) {
                        e = api->Recv(x.ia[par], cnt, ncclFloat32, x.pr * pcol + qk, c->nccl, s);
                    }
                }
                if (cols > 0 && prow > 1 && e == ncclSuccess) {
                    const size_t cnt = ldist::img_floats(cols);
                    if (x.pr == pk) {
                        for (int p = 0; p < prow && e == ncclSuccess; ++p)
                            if (p != pk) e = api->Send(x.ib[par], cnt, ncclFloat32, p * pcol + x.pc, c->nccl, s);
                    } else {
                        e = api->Recv(x.ib[par], cnt, ncclFloat32, pk * pcol + x.pc, c->nccl, s);
                    }
                }
                ncclResult_t e2 = api->GroupEnd();
                if (e == ncclSuccess) e = e2;
                if (e != ncclSuccess) { st = set_error(RODINIA_E_NCCL, "lud_dist panels: %s", api->GetErrorString(e)); goto done; }
            }
        }
        // 4. trailing updates: block row / column k+1 now (main), the rest on the side stream
        LD_CUDA(cudaEventRecord(ev_img, s), "lud_dist event");
        if (rest_pending) LD_CUDA(cudaStreamWaitEvent(s, ev_rest, 0), "lud_dist event");
        LD_CUDA(cudaStreamWaitEvent(s2, ev_img, 0), "lud_dist event");
        {
            const int pn = (int)((k + 1) % prow), qn = (int)((k + 1) % pcol);
            for (auto& x : rk) {
                const int64_t lr0 = bc_blocks_le(k, prow, x.pr) * NB, lc0 = bc_blocks_le(k, pcol, x.pc) * NB;
                const int64_t rows = x.mloc - lr0, cols = x.nloc - lc0;
                if (rows <= 0 || cols <= 0) continue;
                // block row / column k+1 are this rank's first trailing local block row / column
                const int64_t mb = x.pr == pn ? std::min<int64_t>(NB, rows) : 0;
                const int64_t nbk = x.pc == qn ? std::min<int64_t>(NB, cols) : 0;
                const int ga = ldist::img_groups(rows), gb = ldist::img_groups(cols);
                const int next[2][4] = {{(int)lr0, (int)rows, (int)lc0, (int)nbk},                 // column k+1
                                        {(int)lr0, (int)mb, (int)(lc0 + nbk), (int)(cols - nbk)}};  // row k+1
                LD_TRY(ldist::update(x.slot, (int)x.nloc, next, 2, (int)lr0, x.ia[par], ga, (int)lc0, x.ib[par], gb, s, prio_hi));
                const int rest[1][4] = {{(int)(lr0 + mb), (int)(rows - mb), (int)(lc0 + nbk), (int)(cols - nbk)}};
                LD_TRY(ldist::update(x.slot, (int)x.nloc, rest, 1, (int)lr0, x.ia[par], ga, (int)lc0, x.ib[par], gb, s2));
            }
        }
        LD_CUDA(cudaEventRecord(ev_rest, s2), "lud_dist event");
        rest_pending = true;
    }
done:
#undef LD_TRY
#undef LD_CUDA
    cleanup();
    return st;
}

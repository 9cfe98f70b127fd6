// dist.cu -- multi-GPU row-slab decomposition for the stencils (hotspot, srad), one process
// per GPU, NCCL point-to-point halo exchange over NVLink / NVSwitch.
//
// Rank r owns global rows [floor(r*R/P), floor((r+1)*R/P)).  Its local buffer is
//   [top halo][own rows][bottom halo]
// and the kernels clamp neighbours at the *buffer* edges, so the same launch code as the
// single-GPU path runs on a slab: rows next to a non-global buffer edge go stale by one row
// (hotspot; srad: one row at the top, two at the bottom) per step, which the halo depth absorbs.
//  * hotspot: halo D = steps fused per launch (temporal); every D steps each rank sends its
//    first D own rows up and its last D own rows down (ncclSend/ncclRecv in one group on the
//    compute stream).  Power halos are exchanged once.
//  * srad: one iteration reads rows i-1..i+2, so halos are D above and 2D below.  The global
//    ROI statistics q0sqr(t) are computed without any per-iteration collective: every rank
//    gathers the ROI's dependency cone of J0 once (rows [r1-n, r2+2n+2] x cols likewise,
//    ncclBroadcast from the owners) and evolves just that window with the same kernels; ROI
//    values on the window are bit-identical to the full grid (reading S10), hence so is q0sqr(t).
// Results are bitwise identical to the single-GPU call with the same granularity.
//
// A second communicator kind, LOCAL, keeps all P slabs on the current device and moves halos
// with cudaMemcpyAsync; it exercises the identical slab/halo logic on one GPU (tests).
//
// NCCL is not linked: libnccl.so.2 is dlopen'ed at run time (the copy torch already mapped,
// or $RODINIA_NCCL_LIB), so the library loads on hosts without NCCL.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>  // types and enum values only; entry points are resolved with dlsym
#include <string.h>

#include <algorithm>
#include <mutex>
#include <vector>

#include "rg_internal.h"
#include "workloads.h"

struct rodinia_comm {
    int kind;  // 0 = NCCL (one slab per process), 1 = LOCAL (all slabs in this process)
    int nranks, rank;
    ncclComm_t nccl;
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

// ------------------------------------------------------------------ slabs
static void slab_of(int64_t R, int P, int r, int64_t* row0, int64_t* n) {
    const int64_t a = (int64_t)r * R / P, b = (int64_t)(r + 1) * R / P;
    *row0 = a;
    *n = b - a;
}

struct Slab {
    int rank;       // global slab index
    int64_t row0;   // first owned global row
    int own;        // owned rows
    int top, bot;   // halo rows above / below
    float* buf[2];  // local buffers (top + own + bot rows)
    float* aux;     // hotspot: power; unused for srad
    float* scr;     // hotspot: ping-pong scratch for multi-launch periods
    int rows() const { return top + own + bot; }
};

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

static rodinia_status make_slabs(rodinia_comm* c, int64_t R, int up, int down, std::vector<Slab>* out) {
    const int P = c->nranks;
    std::vector<int> ranks;
    if (c->kind == 1)
        for (int r = 0; r < P; ++r) ranks.push_back(r);
    else
        ranks.push_back(c->rank);
    for (int r : ranks) {
        Slab x;
        memset(&x, 0, sizeof x);
        x.rank = r;
        int64_t n;
        slab_of(R, P, r, &x.row0, &n);
        x.own = (int)n;
        x.top = r > 0 ? down : 0;
        x.bot = r + 1 < P ? up : 0;
        if (P > 1 && x.own < std::max(up, down))
            return set_error(RODINIA_E_ILLEGAL_FACTOR,
                             "dist: slab %d has %d rows, fewer than the halo depth %d; use fewer ranks or a "
                             "smaller temporal depth", r, x.own, std::max(up, down));
        out->push_back(x);
    }
    return RODINIA_OK;
}

static void free_slabs(std::vector<Slab>& sl, cudaStream_t s) {
    for (auto& x : sl) {
        scratch_free(x.buf[0], s);
        scratch_free(x.buf[1], s);
        scratch_free(x.aux, s);
        scratch_free(x.scr, s);
    }
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

extern "C" rodinia_status rodinia_comm_destroy(rodinia_comm* c) {
    if (!c) return set_error(RODINIA_E_INVALID, "comm_destroy: null");
    if (c->kind == 0 && c->nccl) {
        NcclApi* api;
        if (nccl_api(&api) == RODINIA_OK) api->CommDestroy(c->nccl);
    }
    delete c;
    return RODINIA_OK;
}

// ===================================================================== exported: hotspot_dist
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
    int64_t row0, own0;
    slab_of(R, c->nranks, 0, &row0, &own0);
    if (!gran_is_zero(g)) gg = *g;
    else {
        rodinia_problem pb{own0, C, iters, c->nranks};
        if (!tune_cache_lookup(RODINIA_HOTSPOT, pb, &gg)) gg = default_gran(RODINIA_HOTSPOT, pb);
    }
    const hotspot::DirectVariant* dv;
    const hotspot::StreamVariant* sv;
    RG_TRY(hotspot::check(gg, own0 + 2 * 64, C, &dv, &sv));
    const int D = hotspot::temporal_of(sv);
    rodinia_hotspot_coeffs cc;
    if (coeffs) cc = *coeffs;
    else rodinia_hotspot_coeffs_rodinia(R, C, 0.016, 0.016, &cc);
    const HsCoef cf = hs_derive(cc.k, cc.rx, cc.ry, cc.rz);  // state form (hs_cell.cuh)
    std::vector<Slab> sl;
    RG_TRY(make_slabs(c, R, D, D, &sl));
    DeviceInfo di;
    RG_TRY(device_info(&di));
    cudaStream_t s = (cudaStream_t)stream;
    const size_t rowb = (size_t)C * sizeof(float);
    rodinia_status st = RODINIA_OK;
    for (size_t i = 0; i < sl.size() && st == RODINIA_OK; ++i) {
        Slab& x = sl[i];
        const size_t bytes = (size_t)x.rows() * rowb;
        st = scratch_alloc((void**)&x.buf[0], bytes, s);
        if (st == RODINIA_OK) st = scratch_alloc((void**)&x.buf[1], bytes, s);
        if (st == RODINIA_OK) st = scratch_alloc((void**)&x.aux, bytes, s);
        if (st == RODINIA_OK) st = scratch_alloc((void**)&x.scr, bytes, s);
        if (st == RODINIA_OK) {
            cudaMemcpyAsync(x.buf[0] + (size_t)x.top * C, arg_ptr(c, temp_local, i), x.own * rowb, cudaMemcpyDeviceToDevice, s);
            cudaMemcpyAsync(x.aux + (size_t)x.top * C, arg_ptr(c, power_local, i), x.own * rowb, cudaMemcpyDeviceToDevice, s);
            // T -> u = T - amb and P -> kP = k*P on the owned rows (halos arrive converted)
            hotspot::convert(x.buf[0] + (size_t)x.top * C, x.buf[0] + (size_t)x.top * C, (int64_t)x.own * C, 0, cc.amb, s);
            hotspot::convert(x.aux + (size_t)x.top * C, x.aux + (size_t)x.top * C, (int64_t)x.own * C, 1, cc.k, s);
        }
    }
    if (st == RODINIA_OK && c->nranks > 1) st = exchange(c, sl, 0, (int)C, D, D, true, s);
    int cur = 0;
    for (int done = 0; st == RODINIA_OK && done < iters;) {
        const int steps = std::min(D, iters - done);
        if (c->nranks > 1) st = exchange(c, sl, cur, (int)C, D, D, false, s);
        for (size_t i = 0; i < sl.size() && st == RODINIA_OK; ++i) {
            Slab& x = sl[i];
            st = hotspot::run(x.buf[cur], x.aux, x.buf[1 - cur], x.scr, x.rows(), (int)C, steps, cf, gg, dv, sv, s);
        }
        cur = 1 - cur;
        done += steps;
    }
    for (size_t i = 0; i < sl.size() && st == RODINIA_OK; ++i) {
        Slab& x = sl[i];
        float* dst = c->kind == 1 ? ((float* const*)out_local)[i] : (float*)out_local;
        hotspot::convert(x.buf[cur] + (size_t)x.top * C, dst, (int64_t)x.own * C, 2, cc.amb, s);  // u -> T
        const cudaError_t ce = cudaGetLastError();
        if (ce != cudaSuccess) st = cuda_error(ce, "hotspot_dist copy-out", __FILE__, __LINE__);
    }
    if (st == RODINIA_OK && cudaGetLastError() != cudaSuccess) st = set_error(RODINIA_E_CUDA, "hotspot_dist: launch failed");
    free_slabs(sl, s);
    return st;
}

// ===================================================================== exported: srad_dist
extern "C" rodinia_status rodinia_srad_dist(rodinia_comm* c, void* J_local, int64_t R, int64_t C, int64_t r1,
                                            int64_t r2, int64_t c1, int64_t c2, float lambda, int32_t niter,
                                            const rodinia_granularity* g, void* stream) {
    if (!c || !J_local) return set_error(RODINIA_E_INVALID, "srad_dist: null argument");
    if (R < 1 || C < 1 || niter < 0 || R < c->nranks) return set_error(RODINIA_E_INVALID, "srad_dist: bad sizes");
    if (r1 < 0 || c1 < 0 || r2 < r1 || c2 < c1 || r2 >= R || c2 >= C)
        return set_error(RODINIA_E_INVALID, "srad_dist: ROI outside the grid");
    if (!std::isfinite(lambda)) return set_error(RODINIA_E_INVALID, "srad_dist: lambda not finite");
    if (c->kind == 1)
        for (int i = 0; i < c->nranks; ++i)
            if (!((float* const*)J_local)[i]) return set_error(RODINIA_E_INVALID, "srad_dist: null slab pointer");
    rodinia_granularity gg;
    int64_t row0, own0;
    slab_of(R, c->nranks, 0, &row0, &own0);
    if (!gran_is_zero(g)) gg = *g;
    else {
        rodinia_problem pb{own0, C, niter, c->nranks};
        if (!tune_cache_lookup(RODINIA_SRAD, pb, &gg)) gg = default_gran(RODINIA_SRAD, pb);
    }
    srad::Plan p;
    RG_TRY(srad::plan(gg, &p));
    if (p.v && p.smem > 48 * 1024)
        RG_CUDA(cudaFuncSetAttribute((const void*)p.v->fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p.smem));
    const int D = 1;  // exchange every iteration (halo 1 row above, 2 below)
    std::vector<Slab> sl;
    RG_TRY(make_slabs(c, R, 2 * D, D, &sl));
    DeviceInfo di;
    RG_TRY(device_info(&di));
    RG_TRY(srad::take_sticky());
    if (niter == 0) return RODINIA_OK;
    cudaStream_t s = (cudaStream_t)stream;
    const size_t rowb = (size_t)C * sizeof(float);
    rodinia_status st = RODINIA_OK;

    // ---- q0sqr(t) from the ROI's dependency cone (no per-iteration collective)
    const int64_t wr0 = std::max<int64_t>(0, r1 - niter), wr1 = std::min<int64_t>(R, r2 + 2 * (int64_t)niter + 3);
    const int64_t wc0 = std::max<int64_t>(0, c1 - niter), wc1 = std::min<int64_t>(C, c2 + 2 * (int64_t)niter + 3);
    const int WR = (int)(wr1 - wr0), WC = (int)(wc1 - wc0);
    float* W = nullptr;
    srad::Engine we;
    RG_TRY(scratch_alloc((void**)&W, (size_t)WR * WC * sizeof(float), s));
    st = srad::engine_alloc(&we, p, WR, WC, niter, s);
    if (st == RODINIA_OK) {
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
    }
    if (st == RODINIA_OK)
        srad::engine_steps(&we, W, we.jb, 0, niter, true, (int)(r1 - wr0), (int)(c1 - wc0), (int)(r2 - r1 + 1),
                           (int)(c2 - c1 + 1), 0.25f * lambda, s);

    // ---- slabs: halo D above, 2D below, exchange every D iterations
    std::vector<srad::Engine> eng(sl.size());
    for (size_t i = 0; i < sl.size() && st == RODINIA_OK; ++i) {
        Slab& x = sl[i];
        st = scratch_alloc((void**)&x.buf[0], (size_t)x.rows() * rowb, s);
        if (st == RODINIA_OK) st = srad::engine_alloc(&eng[i], p, x.rows(), (int)C, niter, s);
        if (st == RODINIA_OK) {
            x.buf[1] = eng[i].jb;
            const float* src = (c->kind == 1 ? ((float* const*)J_local)[i] : (float*)J_local);
            cudaMemcpyAsync(x.buf[0] + (size_t)x.top * C, src, x.own * rowb, cudaMemcpyDeviceToDevice, s);
            cudaMemcpyAsync(eng[i].its, we.its, (size_t)niter * sizeof(SradIter), cudaMemcpyDeviceToDevice, s);
        }
    }
    std::vector<float*> cur(sl.size()), oth(sl.size());
    for (size_t i = 0; i < sl.size(); ++i) { cur[i] = sl[i].buf[0]; oth[i] = sl[i].buf[1]; }
    for (int it = 0; st == RODINIA_OK && it < niter; it += D) {
        if (c->nranks > 1) {
            // exchange on whichever buffer currently holds J (same parity on every slab)
            const int which = (cur[0] == sl[0].buf[0]) ? 0 : 1;
            st = exchange(c, sl, which, (int)C, 2 * D, D, false, s);
        }
        for (size_t i = 0; i < sl.size() && st == RODINIA_OK; ++i) {
            float* res = srad::engine_steps(&eng[i], cur[i], oth[i], it, std::min(niter, it + D), false, 0, 0, 1, 1,
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
    if (st == RODINIA_OK && cudaGetLastError() != cudaSuccess) st = set_error(RODINIA_E_CUDA, "srad_dist: launch failed");
    for (size_t i = 0; i < sl.size(); ++i) {
        scratch_free(sl[i].buf[0], s);
        srad::engine_free(&eng[i], s);
    }
    srad::engine_free(&we, s);
    scratch_free(W, s);
    return st;
}

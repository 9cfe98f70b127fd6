// hotspot3d.cu -- granularity-parameterised hotspot3D (named in PAPER.md:395).
//
// Operation: Rodinia hotspot3D `hotspotOpt1` (readings T1-T4): on an nx x ny x nz grid
// (x fastest) every step computes, with neighbours clamped to the grid,
//   T' = cc*c + cw*W + ce*E + cs*S + cn*N + cb*B + ct*T + sdc*P + ct*amb
// summed left to right in fp32 (products fused into the running sum; ct*amb is the same fp32
// product every step).  All variants call h3_cell(), so they are bit-identical.
//
// h3_direct<TX,TY,MODE>: the original CTA is Rodinia's 64 x 4 threads, one (x, y) column per
// thread, marching up z with the column's B/C/T values in registers (one new load per level).
// Thread coarsening gives each thread TX x TY columns of the 64 x 4 tile (CTA (64/TX) x (4/TY));
// block coarsening merges bx x by tiles per CTA; MODE 1 with TX % 4 == 0 uses 128-bit rows.
// 12 B of HBM per cell-update (read T, read P, write T'); N/S/E/W re-reads hit L1.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <string.h>

#include <vector>

#include "rg_internal.h"

namespace rg {

struct H3Coef {
    float cc, cw, ce, cs, cn, cb, ct, sdc, amb_ct;  // amb_ct = fp32(ct * amb)
};

__device__ __forceinline__ float h3_cell(float c, float w, float e, float s, float n, float b, float t,
                                         float p, const H3Coef& k) {
    float acc = __fmul_rn(k.cc, c);
    acc = __fmaf_rn(k.cw, w, acc);
    acc = __fmaf_rn(k.ce, e, acc);
    acc = __fmaf_rn(k.cs, s, acc);
    acc = __fmaf_rn(k.cn, n, acc);
    acc = __fmaf_rn(k.cb, b, acc);
    acc = __fmaf_rn(k.ct, t, acc);
    acc = __fmaf_rn(k.sdc, p, acc);
    return __fadd_rn(acc, k.amb_ct);
}

template <int TX, int TY, int MODE>
__global__ void __launch_bounds__((64 / TX) * (4 / TY))
    h3_direct(const float* __restrict__ tin, const float* __restrict__ pw, float* __restrict__ tout, int nx,
              int ny, int nz, int bx, int by, H3Coef k) {
    constexpr int NTX = 64 / TX, NTY = 4 / TY;
    const size_t plane = (size_t)nx * ny;
    const int x0 = blockIdx.x * 64 * bx, y0 = blockIdx.y * 4 * by;
    for (int b_y = 0; b_y < by; ++b_y)
#pragma unroll
        for (int t_y = 0; t_y < TY; ++t_y) {
            const int y = y0 + b_y * 4 + (MODE == 0 ? (int)threadIdx.y + t_y * NTY : (int)threadIdx.y * TY + t_y);
            if (y >= ny) continue;
            const int yn = max(y - 1, 0), ys = min(y + 1, ny - 1);
            for (int b_x = 0; b_x < bx; ++b_x) {
                int xs[TX];
#pragma unroll
                for (int t_x = 0; t_x < TX; ++t_x)
                    xs[t_x] = x0 + b_x * 64 + (MODE == 0 ? (int)threadIdx.x + t_x * NTX : (int)threadIdx.x * TX + t_x);
                // column registers: level below / current / above for each of the TX columns
                float cb_[TX], cc_[TX], ct_[TX];
#pragma unroll
                for (int t_x = 0; t_x < TX; ++t_x) {
                    const int x = min(xs[t_x], nx - 1);
                    const size_t i0 = (size_t)y * nx + x;
                    cc_[t_x] = __ldg(tin + i0);
                    cb_[t_x] = cc_[t_x];
                    ct_[t_x] = __ldg(tin + (nz > 1 ? plane : 0) + i0);
                }
                for (int z = 0; z < nz; ++z) {
                    const size_t zo = (size_t)z * plane;
#pragma unroll
                    for (int t_x = 0; t_x < TX; ++t_x) {
                        const int x = xs[t_x];
                        if (x < nx) {
                            const size_t c = zo + (size_t)y * nx + x;
                            const float w = __ldg(tin + zo + (size_t)y * nx + max(x - 1, 0));
                            const float e = __ldg(tin + zo + (size_t)y * nx + min(x + 1, nx - 1));
                            const float s = __ldg(tin + zo + (size_t)ys * nx + x);
                            const float n = __ldg(tin + zo + (size_t)yn * nx + x);
                            tout[c] = h3_cell(cc_[t_x], w, e, s, n, cb_[t_x], ct_[t_x], __ldg(pw + c), k);
                        }
                        // advance the column window
                        const int xc = min(x, nx - 1);
                        cb_[t_x] = cc_[t_x];
                        cc_[t_x] = ct_[t_x];
                        const int zt = min(z + 2, nz - 1);
                        ct_[t_x] = __ldg(tin + (size_t)zt * plane + (size_t)y * nx + xc);
                    }
                }
            }
        }
}

// h3_plane<TX,TY> (flags RODINIA_STREAM): 2.5-D blocking for B200.  A 256-thread CTA owns a
// (32*TX) x (8*TY) tile of (x, y) columns and marches z; each thread keeps its TX x TY cells'
// values at z-1, z, z+1 in registers (B, C, T) and publishes C through a double-buffered
// shared-memory plane whose one-cell halo ring is read from global memory with clamped indices
// (which reproduces the clamped boundary), so N/S/E/W come from shared memory and each plane
// costs one barrier.  HBM per cell-update: T read once (+ halo re-reads from L2), P read, T'
// written.  TX % 4 == 0 moves rows with 128-bit accesses.
template <int TX, int TY>
__global__ void __launch_bounds__(256)
    h3_plane(const float* __restrict__ tin, const float* __restrict__ pw, float* __restrict__ tout, int nx,
             int ny, int nz, int bx, int by, H3Coef k) {
    constexpr int OX = 32 * TX, OY = 8 * TY, SX = OX + 2, SY = OY + 2;
    __shared__ float pl[2][SY][SX + 1];
    const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
    const size_t plane = (size_t)nx * ny;
    const bool vec = (TX % 4 == 0) && ((nx & 3) == 0);
    (void)bx; (void)by;
    const int x0 = blockIdx.x * OX, y0 = blockIdx.y * OY;
    int xs[TX], ys[TY];
#pragma unroll
    for (int i = 0; i < TX; ++i) xs[i] = min(x0 + tx * TX + i, nx - 1);
#pragma unroll
    for (int j = 0; j < TY; ++j) ys[j] = min(y0 + ty * TY + j, ny - 1);
    const bool full_x = x0 + tx * TX + TX <= nx;
    auto load_cells = [&](int z, float (&v)[TY][TX], const float* __restrict__ base) {
        const float* pz = base + (size_t)z * plane;
#pragma unroll
        for (int j = 0; j < TY; ++j) {
            const float* row = pz + (size_t)ys[j] * nx;
            if (vec && full_x) {
#pragma unroll
                for (int q = 0; q < TX / 4; ++q) {
                    const float4 t = __ldg(reinterpret_cast<const float4*>(row + x0 + tx * TX) + q);
                    v[j][(4 * q) % TX] = t.x; v[j][(4 * q + 1) % TX] = t.y;
                    v[j][(4 * q + 2) % TX] = t.z; v[j][(4 * q + 3) % TX] = t.w;
                }
            } else {
#pragma unroll
                for (int i = 0; i < TX; ++i) v[j][i] = __ldg(row + xs[i]);
            }
        }
    };
    float B[TY][TX], Cc[TY][TX], T[TY][TX], P[TY][TX];
    load_cells(0, Cc, tin);
#pragma unroll
    for (int j = 0; j < TY; ++j)
#pragma unroll
        for (int i = 0; i < TX; ++i) B[j][i] = Cc[j][i];
    load_cells(min(1, nz - 1), T, tin);
    load_cells(0, P, pw);
    // halo ring of the tile: left/right columns (SY cells each) and top/bottom rows (OX each);
    // thread t owns ring cells t, t+256, ... and keeps the next plane's values in registers
    constexpr int NHALO = 2 * SY + 2 * OX, NH = (NHALO + 255) / 256;
    int hoff[NH], hsy[NH], hsx[NH];
#pragma unroll
    for (int q = 0; q < NH; ++q) {
        const int h = threadIdx.x + 256 * q;
        int sy = 0, sx = 0;
        if (h < SY) { sy = h; sx = 0; }
        else if (h < 2 * SY) { sy = h - SY; sx = SX - 1; }
        else if (h < 2 * SY + OX) { sy = 0; sx = 1 + (h - 2 * SY); }
        else if (h < NHALO) { sy = SY - 1; sx = 1 + (h - 2 * SY - OX); }
        hsy[q] = sy; hsx[q] = sx;
        const int gy = min(max(y0 - 1 + sy, 0), ny - 1), gx = min(max(x0 - 1 + sx, 0), nx - 1);
        hoff[q] = gy * nx + gx;
    }
    float hv[NH];
#pragma unroll
    for (int q = 0; q < NH; ++q) hv[q] = threadIdx.x + 256 * q < NHALO ? __ldg(tin + hoff[q]) : 0.f;
    for (int z = 0; z < nz; ++z) {
        const int buf = z & 1;
#pragma unroll
        for (int j = 0; j < TY; ++j)
#pragma unroll
            for (int i = 0; i < TX; ++i) pl[buf][1 + ty * TY + j][1 + tx * TX + i] = Cc[j][i];
#pragma unroll
        for (int q = 0; q < NH; ++q)
            if (threadIdx.x + 256 * q < NHALO) pl[buf][hsy[q]][hsx[q]] = hv[q];
        __syncthreads();
        // the next plane's global loads are issued before this plane's arithmetic (one plane of
        // lookahead for T, P and the halo ring), so their latency hides behind the compute
        float T2[TY][TX], P2[TY][TX], hv2[NH];
        const bool more = z + 1 < nz;
        if (more) {
            load_cells(min(z + 2, nz - 1), T2, tin);
            load_cells(z + 1, P2, pw);
            const float* pz1 = tin + (size_t)(z + 1) * plane;
#pragma unroll
            for (int q = 0; q < NH; ++q) hv2[q] = threadIdx.x + 256 * q < NHALO ? __ldg(pz1 + hoff[q]) : 0.f;
        }
#pragma unroll
        for (int j = 0; j < TY; ++j) {
            const int ly = 1 + ty * TY + j;
            const int gy = y0 + ty * TY + j;
            float o[TX];
#pragma unroll
            for (int i = 0; i < TX; ++i) {
                const int lx = 1 + tx * TX + i;
                // clamped halo / interior values; cells beyond the grid edge hold clamped copies
                const float w = (x0 + tx * TX + i == 0) ? Cc[j][i] : pl[buf][ly][lx - 1];
                const float e = (x0 + tx * TX + i >= nx - 1) ? Cc[j][i] : pl[buf][ly][lx + 1];
                const float n = (gy == 0) ? Cc[j][i] : pl[buf][ly - 1][lx];
                const float s_ = (gy >= ny - 1) ? Cc[j][i] : pl[buf][ly + 1][lx];
                o[i] = h3_cell(Cc[j][i], w, e, s_, n, B[j][i], T[j][i], P[j][i], k);
            }
            if (gy < ny) {
                float* orow = tout + (size_t)z * plane + (size_t)gy * nx;
                if (vec && full_x) {
#pragma unroll
                    for (int q = 0; q < TX / 4; ++q)
                        reinterpret_cast<float4*>(orow + x0 + tx * TX)[q] =
                            make_float4(o[(4 * q) % TX], o[(4 * q + 1) % TX], o[(4 * q + 2) % TX], o[(4 * q + 3) % TX]);
                } else {
#pragma unroll
                    for (int i = 0; i < TX; ++i)
                        if (x0 + tx * TX + i < nx) orow[x0 + tx * TX + i] = o[i];
                }
            }
        }
        if (more) {  // advance the z window
#pragma unroll
            for (int j = 0; j < TY; ++j)
#pragma unroll
                for (int i = 0; i < TX; ++i) {
                    B[j][i] = Cc[j][i]; Cc[j][i] = T[j][i]; T[j][i] = T2[j][i]; P[j][i] = P2[j][i];
                }
#pragma unroll
            for (int q = 0; q < NH; ++q) hv[q] = hv2[q];
        }
    }
}

namespace hotspot3d {

typedef void (*Fn)(const float*, const float*, float*, int, int, int, int, int, H3Coef);
struct Variant { int tx, ty, mode; Fn fn; const char* key; };
#define RG_H3(TX, TY, M) {TX, TY, M, h3_direct<TX, TY, M>, "void rg::h3_direct<" #TX ", " #TY ", " #M ">"}
#define RG_H32(TX, TY) RG_H3(TX, TY, 0), RG_H3(TX, TY, 1)
static const Variant kVariants[] = {
    RG_H32(1, 1), RG_H32(2, 1), RG_H32(4, 1), RG_H32(8, 1), RG_H32(1, 2), RG_H32(2, 2), RG_H32(4, 2),
    RG_H32(1, 4), RG_H32(2, 4), RG_H32(4, 4),
};
#undef RG_H32
#undef RG_H3

static const Variant kPlane[] = {
    {1, 1, 1, h3_plane<1, 1>, "void rg::h3_plane<1, 1>"}, {2, 1, 1, h3_plane<2, 1>, "void rg::h3_plane<2, 1>"},
    {4, 1, 1, h3_plane<4, 1>, "void rg::h3_plane<4, 1>"}, {4, 2, 1, h3_plane<4, 2>, "void rg::h3_plane<4, 2>"},
    {2, 2, 1, h3_plane<2, 2>, "void rg::h3_plane<2, 2>"}, {1, 4, 1, h3_plane<1, 4>, "void rg::h3_plane<1, 4>"},
    {4, 4, 1, h3_plane<4, 4>, "void rg::h3_plane<4, 4>"},
};

static const Variant* find(int tx, int ty, int mode, bool plane) {
    if (plane) {
        for (const auto& v : kPlane)
            if (v.tx == tx && v.ty == ty) return &v;
        return nullptr;
    }
    for (const auto& v : kVariants)
        if (v.tx == tx && v.ty == ty && v.mode == mode) return &v;
    return nullptr;
}

rodinia_status check(const rodinia_granularity& g, int64_t ny, const Variant** out) {
    if (g.thread_x < 1 || g.thread_y < 1 || g.block_x < 1 || g.block_y < 1 || g.temporal != 1)
        return set_error(RODINIA_E_ILLEGAL_FACTOR, "hotspot3d: factors >= 1, temporal = 1 (%s)", gran_str(g).c_str());
    if (g.index_mode != 0 && g.index_mode != 1) return set_error(RODINIA_E_ILLEGAL_FACTOR, "hotspot3d: index_mode 0/1");
    const bool plane = (g.flags & RODINIA_STREAM) != 0;
    if (plane) {
        if (g.block_x != 1 || g.block_y != 1 || g.index_mode != 1)
            return set_error(RODINIA_E_NOT_BUILT, "hotspot3d: the plane family has block factors 1, index_mode 1");
        if ((ny + 8 * g.thread_y - 1) / (8 * g.thread_y) > 65535)
            return set_error(RODINIA_E_ILLEGAL_FACTOR, "hotspot3d: grid.y too large");
    } else {
        if (64 % g.thread_x || 4 % g.thread_y)
            return set_error(RODINIA_E_ILLEGAL_FACTOR, "hotspot3d: thread factors must divide the 64 x 4 tile (PAPER.md:237)");
        if (((ny + 3) / 4 + g.block_y - 1) / g.block_y > 65535)
            return set_error(RODINIA_E_ILLEGAL_FACTOR, "hotspot3d: grid.y too large; raise block_y");
    }
    *out = find(g.thread_x, g.thread_y, g.index_mode, plane);
    if (!*out) return set_error(RODINIA_E_NOT_BUILT, "hotspot3d: variant %s not instantiated", gran_str(g).c_str());
    return boundary_filter(RODINIA_HOTSPOT3D, (*out)->key, plane ? 256 : (64 / g.thread_x) * (4 / g.thread_y), 0,
                           g.flags);  // compile-time filter at the boundary
}

int num_variants() { return (int)(sizeof(kVariants) / sizeof(kVariants[0]) + sizeof(kPlane) / sizeof(kPlane[0])); }
void variant_info(int i, rodinia_granularity* g, const void** fn, const char** key, int* threads) {
    const int nd = (int)(sizeof(kVariants) / sizeof(kVariants[0]));
    if (i >= nd) {
        const auto& v = kPlane[i - nd];
        *g = gran(v.tx, v.ty, 1, 1, 1, 1, RODINIA_STREAM);
        *fn = (const void*)v.fn;
        *key = v.key;
        *threads = 256;
        return;
    }
    const auto& v = kVariants[i];
    *g = gran(v.tx, v.ty, 1, 1, 1, v.mode);
    *fn = (const void*)v.fn;
    *key = v.key;
    *threads = (64 / v.tx) * (4 / v.ty);
}

rodinia_status run(const float* tin, const float* p, float* tout, float* scr, int nx, int ny, int nz, int iters,
                   const H3Coef& k, const Variant* v, int bx, int by, cudaStream_t s) {
    const size_t n = (size_t)nx * ny * nz;
    if (iters == 0) {
        RG_CUDA(cudaMemcpyAsync(tout, tin, n * sizeof(float), cudaMemcpyDeviceToDevice, s));
        return RODINIA_OK;
    }
    const bool plane = v->mode == 1 && (v->fn == (Fn)h3_plane<1, 1> || v->fn == (Fn)h3_plane<2, 1> ||
                                         v->fn == (Fn)h3_plane<4, 1> || v->fn == (Fn)h3_plane<4, 2> ||
                                         v->fn == (Fn)h3_plane<2, 2> || v->fn == (Fn)h3_plane<1, 4> ||
                                         v->fn == (Fn)h3_plane<4, 4>);
    dim3 grid = plane ? dim3((nx + 32 * v->tx - 1) / (32 * v->tx), (ny + 8 * v->ty - 1) / (8 * v->ty))
                      : dim3(((nx + 63) / 64 + bx - 1) / bx, ((ny + 3) / 4 + by - 1) / by);
    dim3 block = plane ? dim3(256) : dim3(64 / v->tx, 4 / v->ty);
    const float* src = tin;
    for (int l = 0; l < iters; ++l) {
        float* dst = ((iters - 1 - l) % 2 == 0) ? tout : scr;
        v->fn<<<grid, block, 0, s>>>(src, p, dst, nx, ny, nz, bx, by, k);
        count_launch();
        src = dst;
    }
    RG_CUDA(cudaGetLastError());
    return RODINIA_OK;
}

}  // namespace hotspot3d
}  // namespace rg

using namespace rg;

extern "C" rodinia_status rodinia_hotspot3d_coeffs_rodinia(int64_t nx, int64_t ny, int64_t nz, double chip_w,
                                                           double chip_h, double t_chip,
                                                           rodinia_hotspot3d_coeffs* out) {
    if (nx < 1 || ny < 1 || nz < 1 || !(chip_w > 0) || !(chip_h > 0) || !(t_chip > 0) || !out ||
        !std::isfinite(chip_w) || !std::isfinite(chip_h) || !std::isfinite(t_chip))
        return set_error(RODINIA_E_INVALID, "hotspot3d_coeffs: bad arguments");
    // Rodinia hotspot3D constants (T1)
    const double k_si = 100.0, spec_heat = 1.75e6, factor_chip = 0.5, max_pd = 3.0e6, precision = 0.001;
    const double dx = chip_h / (double)ny, dy = chip_w / (double)nx, dz = t_chip / (double)nz;
    const double cap = factor_chip * spec_heat * t_chip * dx * dy;
    const double Rx = dy / (2.0 * k_si * t_chip * dx), Ry = dx / (2.0 * k_si * t_chip * dy);
    const double Rz = dz / (k_si * dx * dy);
    const double dt = precision / (max_pd / (factor_chip * t_chip * spec_heat));
    const double sdc = dt / cap, ce = sdc / Rx, cn = sdc / Ry, ct = sdc / Rz;
    out->cc = (float)(1.0 - (2.0 * ce + 2.0 * cn + 3.0 * ct));
    out->cw = out->ce = (float)ce;
    out->cs = out->cn = (float)cn;
    out->cb = out->ct = (float)ct;
    out->sdc = (float)sdc;
    out->amb = 80.0f;
    return RODINIA_OK;
}

static rodinia_status h3_validate(const void* tin, const void* p, const void* tout, int64_t nx, int64_t ny,
                                  int64_t nz, int32_t iters, const rodinia_hotspot3d_coeffs* c) {
    if (!tin || !p || !tout) return set_error(RODINIA_E_INVALID, "hotspot3d: null buffer");
    if (nx < 1 || ny < 1 || nz < 1) return set_error(RODINIA_E_INVALID, "hotspot3d: sizes must be >= 1");
    if (nx > (1 << 30) || ny > (1 << 30) || nz > (1 << 30) || nx * ny * nz > (1ll << 38))
        return set_error(RODINIA_E_INVALID, "hotspot3d: grid too large");
    if (iters < 0) return set_error(RODINIA_E_INVALID, "hotspot3d: iterations < 0");
    if (tin == tout) return set_error(RODINIA_E_INVALID, "hotspot3d: temp_out must not alias temp_in");
    if (c) {
        const float* f = &c->cc;
        for (int i = 0; i < 9; ++i)
            if (!std::isfinite(f[i])) return set_error(RODINIA_E_INVALID, "hotspot3d: coefficients must be finite");
    }
    return RODINIA_OK;
}

extern "C" rodinia_status rodinia_hotspot3d(const float* tin, const float* p, float* tout, float* scratch, int64_t nx,
                                            int64_t ny, int64_t nz, int32_t iters,
                                            const rodinia_hotspot3d_coeffs* coeffs, const rodinia_granularity* g,
                                            void* stream) {
    RG_TRY(h3_validate(tin, p, tout, nx, ny, nz, iters, coeffs));
    if (scratch && (scratch == tin || scratch == tout)) return set_error(RODINIA_E_INVALID, "hotspot3d: scratch aliases");
    rodinia_granularity gg;
    if (!gran_is_zero(g)) gg = *g;
    else {
        rodinia_problem pb{ny, nx, iters, 1, (int32_t)nz, 0};
        if (!tune_cache_lookup(RODINIA_HOTSPOT3D, pb, &gg)) gg = default_gran(RODINIA_HOTSPOT3D, pb);
    }
    const hotspot3d::Variant* v;
    RG_TRY(hotspot3d::check(gg, ny, &v));
    rodinia_hotspot3d_coeffs cc;
    if (coeffs) cc = *coeffs;
    else rodinia_hotspot3d_coeffs_rodinia(nx, ny, nz, 0.016, 0.016, 0.0005, &cc);
    const H3Coef k{cc.cc, cc.cw, cc.ce, cc.cs, cc.cn, cc.cb, cc.ct, cc.sdc, cc.ct * cc.amb};
    DeviceInfo di;
    RG_TRY(device_info(&di));
    cudaStream_t s = (cudaStream_t)stream;
    float* scr = scratch;
    if (!scr && iters >= 2) RG_TRY(scratch_alloc((void**)&scr, (size_t)nx * ny * nz * sizeof(float), s));
    rodinia_status st = hotspot3d::run(tin, p, tout, scr, (int)nx, (int)ny, (int)nz, iters, k, v, gg.block_x,
                                       gg.block_y, s);
    if (scr != scratch) scratch_free(scr, s);
    return st;
}

extern "C" rodinia_status rodinia_hotspot3d_host(const float* tin, const float* p, float* tout, int64_t nx, int64_t ny,
                                                 int64_t nz, int32_t iters, const rodinia_hotspot3d_coeffs* coeffs,
                                                 const rodinia_granularity* g, void* stream) {
    RG_TRY(h3_validate(tin, p, tout, nx, ny, nz, iters, coeffs));
    DeviceInfo di;
    RG_TRY(device_info(&di));
    const size_t bytes = (size_t)nx * ny * nz * 4;
    void *dt, *dp, *dout;
    std::lock_guard<std::mutex> lk(host_mutex());  // cached buffers: whole H2D/solve/D2H
    RG_TRY(host_buffer(0, bytes, &dt));
    RG_TRY(host_buffer(1, bytes, &dp));
    RG_TRY(host_buffer(2, bytes, &dout));
    cudaStream_t s = (cudaStream_t)stream;
    RG_CUDA(cudaMemcpyAsync(dt, tin, bytes, cudaMemcpyHostToDevice, s));
    RG_CUDA(cudaMemcpyAsync(dp, p, bytes, cudaMemcpyHostToDevice, s));
    RG_TRY(rodinia_hotspot3d((const float*)dt, (const float*)dp, (float*)dout, nullptr, nx, ny, nz, iters, coeffs, g,
                             stream));
    RG_CUDA(cudaMemcpyAsync(tout, dout, bytes, cudaMemcpyDeviceToHost, s));
    RG_CUDA(cudaStreamSynchronize(s));
    return RODINIA_OK;
}

// ------------------------------------------------------------------ tuner hooks
namespace rg {
int hotspot3d_num_variants() { return hotspot3d::num_variants(); }
void hotspot3d_variant_info(int i, rodinia_granularity* g, const void** fn, const char** key, int* threads) {
    hotspot3d::variant_info(i, g, fn, key, threads);
}

rodinia_status tune_hotspot3d(const rodinia_problem& pr, int reps, rodinia_granularity* best,
                              std::vector<rodinia_tune_row>* rows) {
    const int nx = (int)pr.cols, ny = (int)pr.rows, nz = std::max(1, pr.depth);
    const int iters = std::max(1, std::min(pr.iterations, 10));
    const size_t n = (size_t)nx * ny * nz;
    cudaStream_t s;
    RG_CUDA(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    float *tin = nullptr, *pw = nullptr, *tout = nullptr, *scr = nullptr;
    rodinia_status st = RODINIA_OK;
    if (cudaMalloc(&tin, n * 4) || cudaMalloc(&pw, n * 4) || cudaMalloc(&tout, n * 4) || cudaMalloc(&scr, n * 4)) {
        cudaGetLastError();
        st = set_error(RODINIA_E_NOMEM, "hotspot3d tune: allocation failed");
    }
    if (st == RODINIA_OK) { cudaMemsetAsync(tin, 0, n * 4, s); cudaMemsetAsync(pw, 0, n * 4, s); }
    rodinia_hotspot3d_coeffs cc;
    rodinia_hotspot3d_coeffs_rodinia(nx, ny, nz, 0.016, 0.016, 0.0005, &cc);
    const H3Coef k{cc.cc, cc.cw, cc.ce, cc.cs, cc.cn, cc.cb, cc.ct, cc.sdc, cc.ct * cc.amb};
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best_ms = 1e30f;
    for (int vi = 0; st == RODINIA_OK && vi < hotspot3d::num_variants(); ++vi) {
        for (auto b : {std::make_pair(1, 1), std::make_pair(2, 1), std::make_pair(1, 2), std::make_pair(2, 2),
                       std::make_pair(1, 4)}) {
            if (vi >= (int)(sizeof(hotspot3d::kVariants) / sizeof(hotspot3d::kVariants[0])) && (b.first != 1 || b.second != 1)) continue;
            rodinia_tune_row row;
            memset(&row, 0, sizeof row);
            const void* fn;
            const char* key;
            int threads;
            hotspot3d::variant_info(vi, &row.g, &fn, &key, &threads);
            row.g.block_x = b.first;
            row.g.block_y = b.second;
            row.median_ms = -1.f;
            row.model_ms = -1.f;
            const hotspot3d::Variant* v = nullptr;
            rodinia_status cs = hotspot3d::check(row.g, ny, &v);
            const PtxasStats* ps = find_stats(key);
            row.regs = ps ? ps->regs : -1;
            row.spill_bytes = ps ? ps->spill_stores + ps->spill_loads : -1;
            row.threads = threads;
            if (cs == RODINIA_OK) {
                row.ctas_per_sm = ctas_per_sm(fn, threads, 0);
                cs = filter_decision(ps, threads, 0, 0);
            }
            if (cs == RODINIA_OK) cs = prune_gate(RODINIA_HOTSPOT3D, pr, &row);
            if (cs == RODINIA_OK) {
                std::vector<float> ts;
                for (int r = -1; r < reps && cs == RODINIA_OK; ++r) {
                    cudaEventRecord(e0, s);
                    cs = hotspot3d::run(tin, pw, tout, scr, nx, ny, nz, iters, k, v, row.g.block_x, row.g.block_y, s);
                    cudaEventRecord(e1, s);
                    if (cudaEventSynchronize(e1) != cudaSuccess)
                        st = cs = cuda_error(cudaGetLastError(), "hotspot3d tune", __FILE__, __LINE__);
                    float ms = 0;
                    cudaEventElapsedTime(&ms, e0, e1);
                    if (r >= 0) ts.push_back(ms);
                }
                if (cs == RODINIA_OK) {
                    std::sort(ts.begin(), ts.end());
                    row.median_ms = ts[ts.size() / 2];
                    if (row.median_ms < best_ms) { best_ms = row.median_ms; *best = row.g; }
                }
            }
            row.status = cs;
            rows->push_back(row);
        }
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(tin); cudaFree(pw); cudaFree(tout); cudaFree(scr);
    cudaStreamDestroy(s);
    if (st == RODINIA_OK && best_ms >= 1e29f) st = set_error(RODINIA_E_FILTERED, "hotspot3d tune: no variant survived");
    if (st == RODINIA_OK) tune_cache_store(RODINIA_HOTSPOT3D, pr, *best, best_ms);
    return st;
}
}  // namespace rg

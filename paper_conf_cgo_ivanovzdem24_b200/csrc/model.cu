// model.cu -- heuristic pre-pruning from kernel statistics.
//
// PAPER.md:253-265 lists the statistics the paper's flow can collect per alternative before
// timing: closed-form counts of arithmetic and memory operations, and, after ptxas, register
// usage, spilling and estimated occupancy; PAPER.md:405 leaves heuristics that pick factors
// from them to future work.  This file is that heuristic for the stencil workloads: for a
// granularity it counts, in closed form,
//   * algorithmic HBM bytes, including the halo re-reads the tile shape implies,
//   * issued lane-instructions, including the redundant halo updates of temporal blocking,
//   * launches,
// and turns them into a time with a roofline, max(bytes / BW, instructions / issue rate),
// divided by a latency-hiding factor 1 - exp(-2 resident warps / W_sat) computed from the ptxas
// registers and shared memory (occupancy), times the wave-quantization factor ceil(w)/w of the
// launch's w = CTAs / (CTAs per SM x SMs) waves, plus a fixed cost per launch.  The per-update
// instruction counts are the measured SASS mixes of each family (DESIGN.md §5 "Pre-pruning");
// the model only has to rank candidates, rodinia_tune_pruned times the best-ranked ones.
// lud and pathfinder are not modelled (latency chains: lud's panel graph, pathfinder's 99
// dependent rows) and are always timed.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>

#include "rg_internal.h"

namespace rg {

struct ModelDevice {
    int sms = 148;
    double clk_hz = 1.965e9;      // SM boost clock
    double bw = 6.45e12;          // sustained HBM bytes/s (≈ 0.8 x the pin rate)
    int regs_per_sm = 65536;
    int smem_per_sm = 228 * 1024;
    int max_warps = 64;
    int max_ctas = 32;
};

static ModelDevice model_device() {
    ModelDevice md;
    int cnt = 0;
    if (cudaGetDeviceCount(&cnt) != cudaSuccess || cnt == 0) {
        cudaGetLastError();
        return md;  // B200 nominal values
    }
    int dev = 0, v = 0;
    cudaGetDevice(&dev);
    if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) == cudaSuccess && v > 0) md.sms = v;
    if (cudaDeviceGetAttribute(&v, cudaDevAttrClockRate, dev) == cudaSuccess && v > 0) md.clk_hz = v * 1e3;
    int mclk = 0, bus = 0;
    if (cudaDeviceGetAttribute(&mclk, cudaDevAttrMemoryClockRate, dev) == cudaSuccess &&
        cudaDeviceGetAttribute(&bus, cudaDevAttrGlobalMemoryBusWidth, dev) == cudaSuccess && mclk > 0 && bus > 0)
        md.bw = 0.8 * 2.0 * mclk * 1e3 * bus / 8.0;  // DDR pin rate x measured copy efficiency
    if (cudaDeviceGetAttribute(&v, cudaDevAttrMaxRegistersPerMultiprocessor, dev) == cudaSuccess && v > 0)
        md.regs_per_sm = v;
    if (cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev) == cudaSuccess && v > 0)
        md.smem_per_sm = v;
    cudaGetLastError();
    return md;
}

// CTAs per SM from ptxas statistics (the occupancy calculator's register, shared-memory, warp
// and CTA limits; registers allocated per warp in units of 256).
static int host_ctas_per_sm(int regs, int threads, int smem, const ModelDevice& md) {
    if (threads < 1) return 0;
    const int warps = (threads + 31) / 32;
    int n = std::min(md.max_ctas, md.max_warps / warps);
    if (regs > 0) {
        const int per_warp = ((regs * 32 + 255) / 256) * 256;
        n = std::min(n, md.regs_per_sm / (per_warp * warps));
    }
    if (smem > 0) n = std::min(n, md.smem_per_sm / (smem + 1024));  // 1 KB per CTA reserved
    return std::max(n, 0);
}

namespace {
struct Work {
    double bytes = 0;        // HBM bytes
    double lane_instr = 0;   // issued instructions x active lanes
    double launches = 0;
    double lane_util = 1.0;  // fraction of the 32 lanes a warp-instruction does useful work on
    double w_sat = 32;       // resident warps per SM needed to hide latency
    double ctas = 0;         // CTAs per launch (wave quantization); 0 = many
    bool ok = true;
};
constexpr double kLaunchS = 2.5e-6;  // per-launch cost (launch + tail), measured on B200
// Halo re-reads of neighbouring tiles/bands mostly hit L2 (the neighbours run concurrently):
// ncu on hs_stream<4,8,*> at 16384^2 measured DRAM traffic 1.08x the algorithmic 12 B/cell for
// a staged-read factor of 1.43, i.e. about a quarter of the redundant reads reach HBM.
inline double l2_absorbed(double read_factor) { return 1.0 + 0.27 * (read_factor - 1.0); }
}  // namespace

// ------------------------------------------------------------------------------- hotspot
// direct: per cell 6 FP32 ops of the state form + loads/stores (float4 in contiguous mode with
// TX % 4 == 0: 6 loads + 1 store per 4 cells; else 6 + 1 per cell) + index work amortised over
// the TX x TY cells of a thread.  12 B per cell-update.
// stream (V, H, chunk = 16*by): ⌊iters/H⌋ launches of H steps; a band computes 32V staged
// columns for 32V - 2H output columns, a chunk computes chunk + H - 1 rows per level (the top
// trapezoid), and reads chunk + 2H + 8 rows of T and P (halo + prefetch run-out).  Issued
// instructions per computed update: 6.4 at V = 4 (the ncu mix of hs_stream<4,8,*>: 535 M
// warp-instructions per 16384^2 x 8-step launch, FP32x2 column pairs), 9 at V = 2 (twice the
// shuffles and ring reads per cell; calibrated on the B200 tune table, where <2,8,*> runs 1.5x
// slower than <4,8,*>), 12 at V = 1 (no pairs); W_sat = 8 (OCC 10 and 12 run within noise).  The
// iters % H remainder steps run one per launch at 12 B per update.
static Work hotspot_work(const rodinia_problem& p, const rodinia_granularity& g) {
    Work w;
    const double R = (double)p.rows, C = (double)p.cols, cells = R * C;
    const int iters = std::max(p.iterations, 1);
    if (g.flags & RODINIA_STREAM) {
        const int V = g.thread_x, H = std::max(g.temporal, 1);
        const double chunk = 16.0 * std::max(g.block_y, 1);
        const double sw = 32.0 * V, ow = sw - 2.0 * H;
        if (ow <= 0) { w.ok = false; return w; }
        const int full = iters / H, rem = iters % H;
        const double col_red = sw / ow, row_red = (chunk + H - 1) / chunk;
        const double in_rows = (chunk + 2.0 * H + 8) / chunk;
        // 6 FP32 lane-ops on FP32x2 pairs + per-lane-vector shuffles / shared-memory reads
        const double ipu = V >= 4 ? 6.4 : (V == 2 ? 9.0 : 12.0);
        w.bytes = full * cells * (8.0 * l2_absorbed(col_red * in_rows) + 4.0) + rem * cells * 12.0;
        w.ctas = std::ceil(std::ceil(C / ow) / std::max(g.block_x, 1)) * std::ceil(R / chunk);
        w.lane_instr = full * cells * H * col_red * row_red * ipu + rem * cells * 14.0;
        w.launches = full + rem;
        w.w_sat = 8;  // H levels x V/2 pairs of independent FP32x2 chains per warp
        return w;
    }
    const int tx = g.thread_x, ty = g.thread_y;
    const bool vec = g.index_mode == 1 && tx % 4 == 0;
    const double mem_ops = vec ? 7.0 / 4.0 : 7.0;
    const double ipu = 6.0 + mem_ops + 12.0 / (tx * ty);
    const int threads = (16 / std::max(tx, 1)) * (16 / std::max(ty, 1));  // Rodinia 16x16 tile
    w.bytes = (double)iters * cells * 12.0;
    w.lane_instr = (double)iters * cells * ipu;
    w.launches = iters;
    w.lane_util = std::min(threads, 32) / 32.0;
    w.ctas = std::ceil(C / (16.0 * g.block_x)) * std::ceil(R / (16.0 * g.block_y));
    return w;
}

// ------------------------------------------------------------------------------- srad
// dataflow (uncoarsened): 52 B and ≈ 60 instructions per update, 2 launches per iteration.
// fused (TX, TY, bx, by): J tile (16bx+3) x (16by+3) read per CTA, J written: 4·halo + 4 B;
// ≈ 55 instructions per update + index work.  stream (V, chunk 16*by): band of 32V columns with
// the kernel's halo, chunk + 3 rows read per chunk; 37 instructions per update with column
// pairs (measured srad_stream<4>: 78 M warp-instructions per 8192^2 iteration), 50 unpaired.
// Every iteration adds the ROI statistics launch.
static Work srad_work(const rodinia_problem& p, const rodinia_granularity& g) {
    Work w;
    const double cells = (double)p.rows * p.cols;
    const int iters = std::max(p.iterations, 1);
    if (g.flags & RODINIA_STREAM) {
        const int V = g.thread_x;
        const double sw = 32.0 * V;
        const double ow = sw - (V >= 4 ? 4 : (V == 2 ? 2 : 1)) - (V >= 4 ? 4 : 2);
        const double chunk = 16.0 * std::max(g.block_y, 1);
        if (ow <= 0) { w.ok = false; return w; }
        w.bytes = iters * cells * (4.0 * l2_absorbed((sw / ow) * (chunk + 3) / chunk) + 4.0);
        w.ctas = std::ceil(std::ceil(p.cols / ow) / std::max(g.block_x, 1)) * std::ceil(p.rows / chunk);
        w.lane_instr = iters * cells * (sw / ow) * ((V % 2 == 0) ? 37.0 : 50.0);
        w.launches = 2.0 * iters;
        w.w_sat = 12;
        return w;
    }
    const bool dataflow = g.thread_x == 1 && g.thread_y == 1 && g.block_x == 1 && g.block_y == 1 && g.index_mode == 0;
    if (dataflow) {
        w.bytes = iters * cells * 52.0;
        w.lane_instr = iters * cells * 60.0;
        w.launches = 3.0 * iters;
        return w;
    }
    const double sx = 16.0 * g.block_x, sy = 16.0 * g.block_y;
    const double halo = (sx + 3) * (sy + 3) / (sx * sy);
    const int threads = (16 / g.thread_x) * (16 / g.thread_y);
    w.bytes = iters * cells * (4.0 * l2_absorbed(halo) + 4.0);
    w.lane_instr = iters * cells * (55.0 * halo + 16.0 / (g.thread_x * g.thread_y));
    w.ctas = std::ceil(p.cols / sx) * std::ceil(p.rows / sy);
    w.launches = 2.0 * iters;
    w.lane_util = std::min(threads, 32) / 32.0;
    return w;
}

// ------------------------------------------------------------------------------- hotspot3d
// rows = ny, cols = nx, depth = nz.  12 B per cell-update.  direct (64x4 tile, TX x TY cells per
// thread): ≈ 20 instructions per update + index work, N/S/E/W re-reads from L1, W_sat = 64.  plane (STREAM):
// 256-thread CTAs over (32 TX) x (8 TY) columns with a one-cell halo ring, ≈ 14 per update.
static Work hotspot3d_work(const rodinia_problem& p, const rodinia_granularity& g) {
    Work w;
    const double cells = (double)p.rows * p.cols * std::max(p.depth, 1);
    const int iters = std::max(p.iterations, 1);
    w.launches = iters;
    w.bytes = iters * cells * 12.0;
    if (g.flags & RODINIA_STREAM) {
        const double tx = 32.0 * g.thread_x, ty = 8.0 * g.thread_y;
        const double halo = (tx + 2) * (ty + 2) / (tx * ty);
        w.lane_instr = iters * cells * 14.0 * halo;
        w.w_sat = 16;
        w.ctas = std::ceil(p.cols / tx) * std::ceil(p.rows / ty);
        return w;
    }
    const int threads = (64 / g.thread_x) * (4 / g.thread_y);
    w.lane_instr = iters * cells * (20.0 + 16.0 / (g.thread_x * g.thread_y));
    // each thread marches up z with 4-byte loads: few bytes in flight per warp, so the family
    // needs a full SM of warps to cover HBM latency (measured: 41 % of HBM at 64 warps/SM)
    w.w_sat = 64;
    w.ctas = std::ceil(std::ceil(p.cols / 64.0) / g.block_x) * std::ceil(std::ceil(p.rows / 4.0) / g.block_y);
    w.lane_util = std::min(threads, 32) / 32.0;
    return w;
}

float model_estimate_ms(rodinia_kernel k, const rodinia_problem& p, const rodinia_tune_row& row) {
    Work w;
    switch (k) {
        case RODINIA_HOTSPOT: w = hotspot_work(p, row.g); break;
        case RODINIA_SRAD: w = srad_work(p, row.g); break;
        case RODINIA_HOTSPOT3D: w = hotspot3d_work(p, row.g); break;
        default: return -1.0f;  // lud, pathfinder: not modelled
    }
    if (!w.ok) return -1.0f;
    static const ModelDevice md = model_device();
    int ctas = row.ctas_per_sm > 0 ? row.ctas_per_sm
                                   : host_ctas_per_sm(row.regs, row.threads, std::max(row.smem_bytes, 0), md);
    if (ctas < 1) ctas = 1;
    const double warps = (double)ctas * ((std::max(row.threads, 1) + 31) / 32);
    // latency hiding grows with concurrent useful lanes (sub-warp CTAs count by their active
    // lanes) and saturates: 86 % at W_sat warps, 95 % at 1.5 W_sat
    const double hide = 1.0 - std::exp(-2.0 * warps * w.lane_util / w.w_sat);
    const double issue_rate = md.sms * 128.0 * md.clk_hz;  // 4 schedulers x 32 lanes per SM
    const double t_mem = w.bytes / md.bw;
    const double t_ins = w.lane_instr / (issue_rate * w.lane_util);
    const double spill_pen = row.spill_bytes > 0 ? 1.25 : 1.0;
    // wave quantization: a launch of n CTAs on ctas x SMs slots takes ceil(waves) wave times
    double quant = 1.0;
    if (w.ctas > 0) {
        const double waves = w.ctas / ((double)ctas * md.sms);
        quant = std::ceil(waves) / waves;
    }
    const double t = std::max(t_mem, t_ins) * spill_pen * quant / hide + w.launches * kLaunchS;
    return (float)(t * 1e3);
}

}  // namespace rg

using namespace rg;

extern "C" rodinia_status rodinia_model_ms(rodinia_kernel k, const rodinia_problem* p, rodinia_tune_row* row) {
    if (!p || !row || p->rows < 1 || p->cols < 1 || p->iterations < 0)
        return set_error(RODINIA_E_INVALID, "model: bad arguments");
    if ((int)k < 0 || (int)k > 4) return set_error(RODINIA_E_INVALID, "model: unknown kernel %d", (int)k);
    const rodinia_granularity& g = row->g;
    if (g.thread_x < 1 || g.thread_y < 1 || g.block_x < 1 || g.block_y < 1 || g.temporal < 1)
        return set_error(RODINIA_E_ILLEGAL_FACTOR, "model: factors must be >= 1");
    row->model_ms = model_estimate_ms(k, *p, *row);
    return RODINIA_OK;
}

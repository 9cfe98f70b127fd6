/*
 * rodinia_gran.h -- C ABI of librodinia_gran.so: granularity-parameterised Rodinia kernels
 * (hotspot, srad_v2, pathfinder, lud) for NVIDIA B200 (sm_100a).
 *
 * Source of the operations.  Ivanov et al., "Retargeting and Respecializing GPU Workloads
 * for Performance Portability", CGO'24.  The paper takes
 * existing CUDA kernels (Rodinia v3) and varies their *granularity*: the
 * amount of work per thread (thread coarsening, §V-A) and the amount of
 * work and shared memory per block (block coarsening, §V-B), emitting
 * several alternatives (§VI), pruning them with ptxas register/spill data
 * and choosing one by timing (TDO).  Coarsening never changes
 * what a kernel computes.  Each entry point below therefore takes the
 * plain Rodinia operation plus an explicit rodinia_granularity; DESIGN.md §3 lists every
 * reading of the operations where the paper is silent.
 *
 * Conventions (all entry points):
 *  - Buffers are DEVICE pointers (cudaMalloc / torch CUDA tensors), row-major, C-contiguous,
 *    pitch = cols, owned and freed by the caller, unless the name ends in `_host`, in which
 *    case they are plain host pointers and the call copies in/out itself (synchronous).
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).  Device calls
 *    are stream-ordered: they enqueue work and return; only `_host` calls, rodinia_tune and
 *    rodinia_sync block.
 *  - Errors are returned as rodinia_status, never thrown/aborted.  Argument errors are
 *    detected before any CUDA call (so they are reported on hosts without a GPU too).
 *    Asynchronous kernel faults surface at the next call or at rodinia_sync.
 *    rodinia_last_error() returns a thread-local message for the last non-OK status.
 *  - The library owns only internal scratch (ping-pong / coefficient buffers), allocated
 *    stream-ordered (cudaMallocAsync) and freed stream-ordered before the call returns.
 *  - Sizes are int64_t; rows, cols >= 1.  int32 overflow of pathfinder costs is the
 *    caller's contract (as in Rodinia).
 */
#ifndef RODINIA_GRAN_H
#define RODINIA_GRAN_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define RODINIA_ABI_VERSION 3

typedef enum {
    RODINIA_OK = 0,
    RODINIA_E_INVALID = -1,        /* null pointer, size < 1, iterations < 0, ROI outside grid,
                                      lambda not finite, aliasing in/out buffers            */
    RODINIA_E_ILLEGAL_FACTOR = -2, /* factor < 1; in FAITHFUL mode a thread factor that does not
                                      divide the original tile; temporal depth
                                      larger than the variant/slab supports                   */
    RODINIA_E_SMEM = -3,           /* variant needs more shared memory per CTA than the device
                                      offers (early pruning)                    */
    RODINIA_E_FILTERED = -4,       /* variant rejected by the compile-time ptxas filter: new
                                      spills or < 1 CTA/SM.  Returned by every
                                      entry point for an explicitly requested pruned
                                      instantiation unless flags has RODINIA_FORCE          */
    RODINIA_E_NOT_BUILT = -5,      /* factor combination not instantiated in this build       */
    RODINIA_E_DEGENERATE = -6,     /* srad: ROI mean == 0, q0sqr undefined                     */
    RODINIA_E_NODEV = -7,          /* no CUDA device / driver                                  */
    RODINIA_E_CUDA = -8,           /* CUDA runtime error (message in rodinia_last_error)       */
    RODINIA_E_NCCL = -9,           /* NCCL error or NCCL library not loadable                  */
    RODINIA_E_NOMEM = -10,         /* device or host allocation failed                         */
    RODINIA_E_PRUNED = -11         /* tune row only: ranked below the `keep` best by the kernel-
                                      statistics model of rodinia_tune_pruned, so never timed   */
} rodinia_status;

/* Granularity of one kernel launch (§V).
 *  thread_x/thread_y : thread-coarsening factor -- work units per thread along x / y
 *                      (1 = uncoarsened).  CTA threads = original threads / (tx*ty), number of
 *                      CTAs unchanged.
 *  block_x/block_y   : block-coarsening factor -- original tiles merged into one CTA along
 *                      x / y.  Threads per CTA unchanged, CTAs / (bx*by), shared memory x b
 *                      (PAPER.md:185, 233).  Any value >= 1: remainder tiles are masked in
 *                      the last CTA row/column (the paper's epilogue kernel).
 *  temporal          : time steps fused per launch (hotspot / pathfinder pyramid height,
 *                      srad fused depth); 1 = one step per launch.
 *  index_mode        : 0 = coalescing-friendly (a thread's units are strided by the thread
 *                      count, Fig.11 of the paper), 1 = contiguous (a thread's units are
 *                      adjacent; 4 contiguous fp32 = one 128-bit access).
 *  flags             : bit0 RODINIA_FAITHFUL -- paper factor rules only (thread factors must
 *                      divide the original tile).
 *                      bit1 RODINIA_STREAM -- use the streaming temporal-blocking family
 *                      (hotspot).
 *                      bit2 RODINIA_FORCE -- run the instantiation even if the compile-time
 *                      ptxas filter pruned it (new spills / 0 CTAs per SM);
 *                      without it such a call returns RODINIA_E_FILTERED before any launch.
 *                      bits 8..15 RODINIA_OCC(n) -- register budget of the instantiation:
 *                      target n resident CTAs per SM (launch bounds => <= 65536/(threads*n)
 *                      registers per thread); 0 = the family's preferred instantiation.  This
 *                      is the register/occupancy trade-off the paper can only observe through
 *                      ptxas; here it is an explicit alternative.
 * A NULL rodinia_granularity* (or all fields zero) selects the tuned variant from the tune
 * cache if one exists for this (device, kernel, shape), else the built-in default. */
typedef struct {
    int32_t thread_x, thread_y;
    int32_t block_x, block_y;
    int32_t temporal;
    int32_t index_mode;
    int32_t flags;
} rodinia_granularity;

#define RODINIA_FAITHFUL 1
#define RODINIA_STREAM 2
#define RODINIA_FORCE 4
#define RODINIA_OCC(n) (((n) & 0xff) << 8)
#define RODINIA_OCC_OF(flags) (((flags) >> 8) & 0xff)

typedef enum {
    RODINIA_HOTSPOT = 0, RODINIA_SRAD = 1, RODINIA_PATHFINDER = 2, RODINIA_LUD = 3, RODINIA_HOTSPOT3D = 4
} rodinia_kernel;

/* ---------------------------------------------------------------------------------------
 * hotspot -- Rodinia hotspot `calculate_temp` (2-D thermal RC stencil), see DESIGN.md §3 H1-H8.
 * One step, every cell (clamped neighbours, Jacobi):
 *   T'[i][j] = c + k*( P[i][j] + ((S+N) - 2c)*ry + ((E+W) - 2c)*rx + (amb - c)*rz ),
 *   c = T[i][j], N/S/W/E = T[i-+1][j], T[i][j-+1] clamped to the grid.
 * `k, rx, ry, rz, amb` are explicit (reading H1: Rodinia's fixed 16 mm chip makes the step
 * unstable above ~1386^2 cells).  k = step/Cap, r* = 1/R*.
 */
typedef struct { float k, rx, ry, rz, amb; } rodinia_hotspot_coeffs;

/* Rodinia's chip formulas (H1) in fp64 for a chip_w x chip_h metre die, each
 * coefficient rounded to fp32 once.  Pure host arithmetic. */
rodinia_status rodinia_hotspot_coeffs_rodinia(int64_t rows, int64_t cols, double chip_w_m,
                                              double chip_h_m, rodinia_hotspot_coeffs* out);

/* `iterations` steps from temp_in (never written) into temp_out (must not alias temp_in).
 * power: rows x cols.  scratch: NULL or a rows*cols fp32 device buffer used as the
 * ping-pong partner (else allocated stream-ordered).  coeffs NULL => Rodinia 16 mm chip.
 * iterations == 0 copies temp_in to temp_out. */
rodinia_status rodinia_hotspot(const float* temp_in, const float* power, float* temp_out,
                               float* scratch, int64_t rows, int64_t cols, int32_t iterations,
                               const rodinia_hotspot_coeffs* coeffs,
                               const rodinia_granularity* g, void* stream);

/* Same with HOST buffers: H2D copy of temp_in and power, the solve, D2H copy of the result,
 * all inside the call (synchronous).  Device buffers are cached inside the library. */
rodinia_status rodinia_hotspot_host(const float* temp_in, const float* power, float* temp_out,
                                    int64_t rows, int64_t cols, int32_t iterations,
                                    const rodinia_hotspot_coeffs* coeffs,
                                    const rodinia_granularity* g, void* stream);

/* A batch of `count` independent problems with HOST buffers: problem i reads temp_in[i] and
 * power[i] and writes temp_out[i] (each rows x cols; arrays of `count` host pointers).  Two
 * library-owned device buffer sets are pipelined: the H2D copies of problem i+1 and the D2H
 * copy of problem i-1 run on copy streams while problem i is solved on `stream` (events
 * order reuse of a set).  Synchronous: returns when every result is in host memory.  The
 * copies overlap compute only if the host buffers are pinned.  Per problem the arithmetic is
 * exactly rodinia_hotspot's. */
rodinia_status rodinia_hotspot_host_batch(const float* const* temp_in, const float* const* power,
                                          float* const* temp_out, int32_t count, int64_t rows,
                                          int64_t cols, int32_t iterations,
                                          const rodinia_hotspot_coeffs* coeffs,
                                          const rodinia_granularity* g, void* stream);

/* ---------------------------------------------------------------------------------------
 * hotspot3d -- Rodinia hotspot3D `hotspotOpt1` (7-point 3-D thermal stencil, named in
 * PAPER.md:395), readings T1-T4.  Grid nx (x, fastest) x ny x nz,
 * index z*nx*ny + y*nx + x.  One step, every cell, neighbours clamped to the grid:
 *   T' = cc*c + cw*W + ce*E + cs*S + cn*N + cb*B + ct*T + sdc*P + ct*amb
 * (W/E: x-+1, N/S: y-+1, B/T: z-+1), summed left to right in fp32. */
typedef struct { float cc, cw, ce, cs, cn, cb, ct, sdc, amb; } rodinia_hotspot3d_coeffs;

/* Rodinia's chip formulas (fp64, rounded once): dx = chip_h/ny, dy = chip_w/nx, dz = t_chip/nz,
 * sdc = dt/Cap, ce = cw = sdc/Rx, cn = cs = sdc/Ry, ct = cb = sdc/Rz, cc = 1 - (2ce+2cn+3ct). */
rodinia_status rodinia_hotspot3d_coeffs_rodinia(int64_t nx, int64_t ny, int64_t nz, double chip_w_m,
                                                double chip_h_m, double t_chip_m,
                                                rodinia_hotspot3d_coeffs* out);

/* `iterations` steps from temp_in (never written) into temp_out; power nx*ny*nz; scratch NULL or
 * an nx*ny*nz buffer; coeffs NULL => Rodinia's 16 mm x 16 mm x 0.5 mm chip. */
rodinia_status rodinia_hotspot3d(const float* temp_in, const float* power, float* temp_out,
                                 float* scratch, int64_t nx, int64_t ny, int64_t nz,
                                 int32_t iterations, const rodinia_hotspot3d_coeffs* coeffs,
                                 const rodinia_granularity* g, void* stream);
rodinia_status rodinia_hotspot3d_host(const float* temp_in, const float* power, float* temp_out,
                                      int64_t nx, int64_t ny, int64_t nz, int32_t iterations,
                                      const rodinia_hotspot3d_coeffs* coeffs,
                                      const rodinia_granularity* g, void* stream);

/* ---------------------------------------------------------------------------------------
 * srad_v2 -- Rodinia srad_v2 (speckle-reducing anisotropic diffusion), DESIGN.md §3 S1-S9.
 * Per iteration: q0sqr = var/mean^2 of J over the ROI rows r1..r2, cols c1..c2 (inclusive),
 * summed in fp64, rounded to fp32 once; pass 1 computes the clamped diffusion coefficient c
 * of every cell from the old J; pass 2 updates J += 0.25*lambda*(c*dN + c_S*dS + c*dW +
 * c_E*dE) (Jacobi).  J (rows x cols, values > 0) is updated in place.
 * Returns RODINIA_E_DEGENERATE if the ROI mean becomes 0 (checked on the device; reported at
 * the next call / rodinia_sync as the sticky status, J left as of the failing iteration).
 */
rodinia_status rodinia_srad(float* J, int64_t rows, int64_t cols, int64_t r1, int64_t r2,
                            int64_t c1, int64_t c2, float lambda, int32_t niter,
                            const rodinia_granularity* g, void* stream);
rodinia_status rodinia_srad_host(float* J, int64_t rows, int64_t cols, int64_t r1, int64_t r2,
                                 int64_t c1, int64_t c2, float lambda, int32_t niter,
                                 const rodinia_granularity* g, void* stream);

/* srad_v1 -- Rodinia srad_v1, the srad variant the paper evaluates, DESIGN.md
 * readings V1-V4: extract J = exp(image/255); niter iterations of the srad arithmetic above with
 * the statistics over the WHOLE image (srad_v1's ROI); compress image = log(J)*255.  image
 * (rows x cols, pixel values in [0, 255], row-major) is updated in place.  Same granularity space
 * as rodinia_srad. */
rodinia_status rodinia_srad_v1(float* image, int64_t rows, int64_t cols, float lambda,
                               int32_t niter, const rodinia_granularity* g, void* stream);
rodinia_status rodinia_srad_v1_host(float* image, int64_t rows, int64_t cols, float lambda,
                                    int32_t niter, const rodinia_granularity* g, void* stream);

/* ---------------------------------------------------------------------------------------
 * pathfinder -- Rodinia pathfinder `dynproc_kernel` (min-cost path DP), P1-P6.
 *   prev = wall[0]; next[j] = wall[r][j] + min(prev[j-1], prev[j], prev[j+1]) (existing
 *   indices), r = 1..rows-1; result (cols int32) = prev after the last row.  Bit-exact. */
rodinia_status rodinia_pathfinder(const int32_t* wall, int64_t rows, int64_t cols,
                                  int32_t* result, const rodinia_granularity* g, void* stream);
rodinia_status rodinia_pathfinder_host(const int32_t* wall, int64_t rows, int64_t cols,
                                       int32_t* result, const rodinia_granularity* g,
                                       void* stream);

/* ---------------------------------------------------------------------------------------
 * lud -- Rodinia lud (blocked Doolittle LU, no pivoting), L1-L6.  a (n x n fp32)
 * is factored in place: unit-diagonal L strictly below the diagonal, U on and above.
 * panel: block (panel) width; 16 = Rodinia's BLOCK_SIZE (0 => 16).  Supported: 16, 32, and
 * 128: per 128-wide block column the diagonal block is factored by one CTA, L21 / U12 are solved
 * one thread per row / column, and the rank-128 trailing update runs on the tensor cores
 * (tcgen05.mma kind::tf32 with the 3xTF32 split; g is ignored there); its
 * quotients are IEEE quotients formed from the pivot's correctly rounded reciprocal.  While at
 * least n/2 rows remain, two block columns share one rank-256 remainder update (environment
 * RG_LUD_PAIR = the row threshold, 0 = off; it changes the rounding order of those updates).
 * The panel width changes fp32 rounding order and is reported separately from coarsening
 * (reading L5).  Zero pivots give inf/NaN (no pivoting, as Rodinia). */
rodinia_status rodinia_lud(float* a, int64_t n, int32_t panel, const rodinia_granularity* g,
                           void* stream);
rodinia_status rodinia_lud_host(float* a, int64_t n, int32_t panel,
                                const rodinia_granularity* g, void* stream);

/* ---------------------------------------------------------------------------------------
 * Variants, compile-time filter and timing-driven tuning (§VI, 251-269).
 */
typedef struct {
    int64_t rows, cols;      /* lud: rows = cols = n; pathfinder: rows x cols wall;
                                hotspot3d: rows = ny, cols = nx (depth = nz) */
    int32_t iterations;      /* hotspot / srad iterations (tuning times a prefix of them);
                                lud: the panel width (0 => 16); pathfinder: unused */
    int32_t nranks;          /* 1 for single-GPU problems; part of the cache key */
    int32_t depth;           /* hotspot3d: nz (0 => 1); others: 0 */
    int32_t reserved;        /* 0 */
} rodinia_problem;

typedef struct {
    rodinia_granularity g;
    float median_ms;         /* tune rows only; -1 when not timed */
    int32_t regs;            /* registers / thread (ptxas) */
    int32_t spill_bytes;     /* spill stores + loads (ptxas) */
    int32_t smem_bytes;      /* static + dynamic shared memory per CTA at this shape */
    int32_t threads;         /* threads per CTA */
    int32_t ctas_per_sm;     /* occupancy (runtime query; 0 when no device) */
    int32_t status;          /* RODINIA_OK, or why the variant is pruned */
    float model_ms;          /* kernel-statistics model estimate (rodinia_model_ms); -1 when the
                                workload is not modelled or the row was not ranked */
} rodinia_tune_row;

/* Enumerate the instantiated variants of kernel k with their ptxas statistics and the
 * compile-time filter decision.  *n: in = capacity of out (may be 0), out = number of
 * variants.  Pure host call (no device needed). */
rodinia_status rodinia_variants(rodinia_kernel k, rodinia_tune_row* out, int32_t* n);

/* Time every surviving variant on synthetic inputs of the problem's shape (never the
 * caller's buffers): `reps` timed runs after one warm-up, CUDA events, median, argmin.
 * Writes the winner to *best and stores it in the tune cache ($RODINIA_TUNE_CACHE, JSON
 * lines, keyed by device name, SM count, kernel, shape, nranks).  rows/nrows as above. */
rodinia_status rodinia_tune(rodinia_kernel k, const rodinia_problem* p, int32_t reps,
                            rodinia_granularity* best, rodinia_tune_row* rows,
                            int32_t* nrows);

/* Heuristic pre-pruning ("kernel statistics", the factor
 * heuristics the paper leaves to future work).  Same as rodinia_tune, but every
 * candidate that survives the compile-time filter is first ranked by rodinia_model_ms and only
 * the `keep` best-ranked are timed; the others come back with status RODINIA_E_PRUNED and their
 * model_ms.  Candidates the model cannot estimate (model_ms < 0: lud, pathfinder) are always
 * timed.  keep <= 0 times every candidate (= rodinia_tune).  For hotspot the candidate set is
 * the tuner's stage-2 block-factor sweep over every instantiation, not only the stage-1 top 4. */
rodinia_status rodinia_tune_pruned(rodinia_kernel k, const rodinia_problem* p, int32_t reps,
                                   int32_t keep, rodinia_granularity* best, rodinia_tune_row* rows,
                                   int32_t* nrows);

/* The model behind rodinia_tune_pruned, host-only (no device needed): estimates the time of one
 * call of kernel k on problem p at row->g from closed-form work counts of the granularity
 * (algorithmic HBM bytes incl. halo redundancy, issued lane-instructions incl. redundant halo
 * updates, launches) and the ptxas statistics of the instantiation (registers, shared memory ->
 * CTAs per SM -> latency-hiding factor), as a roofline max(bytes/BW, instructions/issue rate)
 * divided by the occupancy factor plus a per-launch cost (DESIGN.md §5 "Pre-pruning").
 * row->g, threads, regs, smem_bytes are inputs (ctas_per_sm too when > 0, else it is derived
 * from regs/smem/threads); writes row->model_ms (-1 when the workload is not modelled).
 * Device constants come from the current device when one exists, else B200 nominal values. */
rodinia_status rodinia_model_ms(rodinia_kernel k, const rodinia_problem* p, rodinia_tune_row* row);

/* Resolve what a NULL/zero granularity would run for this problem (cache or default). */
rodinia_status rodinia_resolve(rodinia_kernel k, const rodinia_problem* p,
                               rodinia_granularity* out);

/* ---------------------------------------------------------------------------------------
 * Multi-GPU row-slab decomposition (hotspot, srad), one process per GPU.  The NCCL
 * communicator is bootstrapped from a unique id the caller distributes (e.g. with
 * torch.distributed.broadcast_object_list).  NCCL is loaded at run time (dlopen of the
 * libnccl.so.2 already mapped by torch, else $RODINIA_NCCL_LIB).
 * Rank r owns global rows [floor(r*R/P), floor((r+1)*R/P)).
 */
typedef struct rodinia_comm rodinia_comm;

rodinia_status rodinia_slab(int64_t global_rows, int32_t nranks, int32_t rank, int64_t* row0,
                            int64_t* nrows);
rodinia_status rodinia_comm_unique_id(uint8_t id[128]);
rodinia_status rodinia_comm_init(rodinia_comm** out, int32_t nranks, int32_t rank,
                                 const uint8_t id[128]);
/* In-process "loopback" communicator: `nranks` slabs on the current device, halos moved
 * with cudaMemcpyAsync (tests the decomposition on one GPU). */
rodinia_status rodinia_comm_init_local(rodinia_comm** out, int32_t nranks);
rodinia_status rodinia_comm_destroy(rodinia_comm* comm);

/* The schedule a rank follows (host only, no device needed):
 *  row0, own          owned global rows [row0, row0 + own) (= rodinia_slab)
 *  top, bot           halo rows stored above / below the owned rows
 *  period             iterations between halo exchanges (the temporal depth D)
 *  send_up, send_down rows sent per exchange to rank-1 (its first owned rows) / rank+1 (its last)
 *  exchanges          exchanges in `iterations` (0 for one rank)
 *  overlap            1 if the interior launch of a period overlaps its exchange (hotspot)
 *  cone_*             srad: the ROI's dependency-cone window [cone_r0, cone_r1) x [cone_c0,
 *                     cone_c1) every rank evolves to obtain q0sqr(t) (reading S10); 0 for hotspot
 * hotspot: D = steps per launch of the granularity, halos D / D, sends D / D.
 * srad: D = granularity temporal (a NULL/zero granularity: min(8, rows per slab / 2)), halos D
 * above / 2D below (one iteration reads rows i-1..i+2), sends 2D up / D down.
 * r1..c2: the srad ROI (ignored for hotspot).  Errors: RODINIA_E_INVALID (arguments, other
 * kernels: pathfinder is replicas only, lud has its own 2-D block-cyclic rodinia_lud_dist),
 * RODINIA_E_ILLEGAL_FACTOR (slab thinner than the
 * halo), granularity errors as for the single-GPU call. */
typedef struct {
    int64_t row0, own;
    int32_t top, bot;
    int32_t period;
    int32_t send_up, send_down;
    int32_t exchanges;
    int32_t overlap;
    int32_t reserved;
    int64_t cone_r0, cone_r1, cone_c0, cone_c1;
} rodinia_dist_plan;
rodinia_status rodinia_dist_schedule(rodinia_kernel k, int64_t global_rows, int64_t cols, int32_t nranks,
                                 int32_t rank, int32_t iterations, int64_t r1, int64_t r2, int64_t c1,
                                 int64_t c2, const rodinia_granularity* g, rodinia_dist_plan* out);

/* NCCL communicator: temp_local/power_local/out_local hold this rank's slab (rodinia_slab
 * rows x cols).  Local communicator: the pointers are arrays of `nranks` slab pointers
 * (const float* const*), passed as the same arguments.  Bitwise equal to rodinia_hotspot
 * on the whole grid with the same granularity. */
rodinia_status rodinia_hotspot_dist(rodinia_comm* comm, const void* temp_local,
                                    const void* power_local, void* out_local,
                                    int64_t global_rows, int64_t cols, int32_t iterations,
                                    const rodinia_hotspot_coeffs* coeffs,
                                    const rodinia_granularity* g, void* stream);
/* srad on row slabs: J_local is this rank's slab (LOCAL: array of slab pointers), updated in
 * place; g->temporal (>= 1) is the exchange period D (each launch is still one iteration), a
 * NULL/zero granularity picks the tuned kernel and D = min(8, rows per slab / 2).  Bitwise equal
 * to rodinia_srad on the whole grid with the same kernel granularity. */
rodinia_status rodinia_srad_dist(rodinia_comm* comm, void* J_local, int64_t global_rows,
                                 int64_t cols, int64_t r1, int64_t r2, int64_t c1, int64_t c2,
                                 float lambda, int32_t niter, const rodinia_granularity* g,
                                 void* stream);

/* 2-D block-cyclic multi-GPU LU (the last step).  The same
 * operation as rodinia_lud (Doolittle, no pivoting, packed in place; DESIGN.md §3 L1-L6) on a
 * prow x pcol process grid, rank r = pr * pcol + pc, blocks of NB = 128: global block (I, J)
 * (rows [128 I, 128 I + 128) x cols [128 J, ...), the last ones partial) lives on rank
 * (I mod prow, J mod pcol).  a_local: this rank's local matrix (LOCAL communicator: an array of
 * `nranks` local-matrix pointers, rank order), device, row-major, mloc x nloc with leading
 * dimension nloc (rodinia_lud_dist_layout): the rank's block rows in increasing I by its block
 * columns in increasing J.  Factored in place.  Per block column k: the owner of A_kk factors
 * it and broadcasts it (ncclBroadcast; LOCAL: copies), process column k mod pcol solves
 * L_Ik = A_Ik U_kk^-1, process row k mod prow solves U_kJ = L_kk^-1 A_kJ, the L panels travel
 * along process rows and the U panels along process columns (ncclSend/ncclRecv, as hi/lo TF32
 * operand images), and every rank applies A_IJ -= L_Ik U_kJ to its trailing blocks on the tensor
 * cores (3xTF32, the panel-128 update).  Per element the arithmetic does not depend on the grid:
 * every grid (1 x 1 included) gives the same bits.  Stream-ordered on `stream`; scratch is
 * stream-ordered (cudaMallocAsync) and released at the end.  Errors: RODINIA_E_INVALID (grid
 * != nranks, null pointers), RODINIA_E_NOMEM, RODINIA_E_NCCL, RODINIA_E_CUDA. */
rodinia_status rodinia_lud_dist(rodinia_comm* comm, void* a_local, int64_t n, int32_t prow, int32_t pcol,
                                void* stream);
/* Host only: local matrix shape (rows mloc, columns nloc) of `rank` for rodinia_lud_dist. */
rodinia_status rodinia_lud_dist_layout(int64_t n, int32_t prow, int32_t pcol, int32_t rank, int64_t* mloc,
                                       int64_t* nloc);

/* Split a *total* coarsening factor over `ndims` (1..3) dimensions (footnote 4,
 * "for a total factor of 16, we will coarsen the 3 dimensions with 4, 2, and 2
 * respectively, whereas for 6 we will coarsen with 3, 2, and 1").  Reading G3: the prime factors
 * of `total`, largest first, each go to the dimension with the smallest current factor (x wins
 * ties).  Pure host call; out[0..2] receives the x, y, z factors (1 for unused dimensions). */
rodinia_status rodinia_split_total(int32_t total, int32_t ndims, int32_t out[3]);

/* ---------------------------------------------------------------------------------------
 * Misc. */
const char* rodinia_last_error(void);
const char* rodinia_status_string(rodinia_status s);
rodinia_status rodinia_sync(void* stream);          /* stream sync + sticky async errors */
int32_t rodinia_abi_version(void);
/* Number of kernel launches this library has issued since load (for bench accounting). */
int64_t rodinia_launch_count(void);
/* Dominant-kernel timing (bench roofline).  enable != 0 starts recording a CUDA
 * event pair around every stepping launch of hotspot (hs_stream / hs_direct) on the caller's
 * stream and clears earlier records; enable == 0 stops.  rodinia_kernel_time() synchronises on
 * the recorded events and returns the summed elapsed milliseconds and the number of timed
 * launches since the last enable.  Host-only bookkeeping; errors: RODINIA_E_CUDA. */
rodinia_status rodinia_kernel_timing(int32_t enable);
rodinia_status rodinia_kernel_time(double* total_ms, int64_t* launches);

#ifdef __cplusplus
}
#endif
#endif /* RODINIA_GRAN_H */

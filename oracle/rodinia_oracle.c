/*
 * rodinia_oracle.c -- plain, slow, obviously-correct CPU oracle for the four workloads
 * whose granularity the paper varies (hotspot, srad_v2, pathfinder, lud).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_conf_cgo_ivanovzdem24_b200, librodinia_gran.so) never links, imports or calls
 * it, and this file includes nothing from the product (no shared headers, helpers or
 * constants).
 *
 * Why these definitions: the paper (Ivanov et al., CGO'24, /root/reference/PAPER.md)
 * transforms *existing* Rodinia v3 CUDA kernels (ref [21] PAPER.md:692) and
 * states that coarsening never changes what a kernel computes -- unroll-and-interleave
 * preserves the order of side effects within an iteration (§IV) and the
 * authors verify results by comparing outputs across configurations (PAPER.md:295,
 * §VII-A).  The paper itself prints no kernel formula, so each function below writes out
 * the plain, uncoarsened, iteration-by-iteration definition of the Rodinia kernel it
 * names, in fp64 (the paper fixes no precision) and in the order the definition states.
 * Every reading where the paper is silent is listed in DESIGN.md §3 ("Readings").
 *
 * Build: gcc -O2 -std=c99 -ffp-contract=off -fPIC -shared (no fast-math).
 * Single-threaded, deterministic.  A second build with -fopenmp (liboracle_omp.so) spreads the
 * independent per-cell loops of the stencil steps (hotspot, srad passes 1/2, pathfinder's row,
 * hotspot3D) over threads for the CPU baseline on the GPU box's cores; every
 * cell's arithmetic and every reduction (the ROI sums, lud) are unchanged and sequential, so
 * both builds return identical bits.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORACLE_OK 0
#define ORACLE_EINVAL (-1)
#define ORACLE_EDEGENERATE (-6)
#define ORACLE_ENOMEM (-10)

#ifdef _OPENMP
#include <omp.h>
#define ORACLE_PAR _Pragma("omp parallel for schedule(static)")
#else
#define ORACLE_PAR
#endif

/* Threads used by the per-cell loops (OpenMP build); returns the count in effect (1 without
 * OpenMP). */
int oracle_set_threads(int n) {
#ifdef _OPENMP
    if (n >= 1) omp_set_num_threads(n);
    return omp_get_max_threads();
#else
    (void)n;
    return 1;
#endif
}

static long lmin(long a, long b) { return a < b ? a : b; }
static long lmax(long a, long b) { return a > b ? a : b; }

/* ------------------------------------------------------------------------------------ */
/* hotspot (Rodinia hotspot `calculate_temp` / `compute_tran_temp`; reading H1-H7)
 *
 * Chip-derived coefficients.  Rodinia's constants: t_chip = 0.0005 m, K_SI = 100,
 * SPEC_HEAT_SI = 1.75e6, FACTOR_CHIP = 0.5, MAX_PD = 3.0e6, PRECISION = 0.001, amb = 80.
 * grid cell gw = chip_w/cols, gh = chip_h/rows.
 *   Cap = FACTOR_CHIP*SPEC_HEAT_SI*t_chip*gw*gh
 *   Rx  = gw / (2*K_SI*t_chip*gh);  Ry = gh / (2*K_SI*t_chip*gw);  Rz = t_chip/(K_SI*gh*gw)
 *   step = PRECISION / (MAX_PD / (FACTOR_CHIP*t_chip*SPEC_HEAT_SI))
 * The update uses k = step/Cap and the conductances rx = 1/Rx, ry = 1/Ry, rz = 1/Rz.
 * out[0..4] = {k, rx, ry, rz, amb}.
 */
int oracle_hotspot_coeffs_rodinia(long rows, long cols, double chip_w, double chip_h,
                                  double out[5]) {
    if (rows < 1 || cols < 1 || !(chip_w > 0) || !(chip_h > 0) || !out) return ORACLE_EINVAL;
    const double t_chip = 0.0005, k_si = 100.0, spec_heat_si = 1.75e6;
    const double factor_chip = 0.5, max_pd = 3.0e6, precision = 0.001, amb = 80.0;
    double gw = chip_w / (double)cols;
    double gh = chip_h / (double)rows;
    double cap = factor_chip * spec_heat_si * t_chip * gw * gh;
    double rx = gw / (2.0 * k_si * t_chip * gh);
    double ry = gh / (2.0 * k_si * t_chip * gw);
    double rz = t_chip / (k_si * gh * gw);
    double max_slope = max_pd / (factor_chip * t_chip * spec_heat_si);
    double step = precision / max_slope;
    out[0] = step / cap;
    out[1] = 1.0 / rx;
    out[2] = 1.0 / ry;
    out[3] = 1.0 / rz;
    out[4] = amb;
    return ORACLE_OK;
}

/* One explicit (Jacobi) step of the 2-D thermal RC stencil, every cell:
 *   c = T[i][j]; N = T[max(i-1,0)][j]; S = T[min(i+1,R-1)][j];
 *   W = T[i][max(j-1,0)]; E = T[i][min(j+1,C-1)]                 (clamped = adiabatic edge)
 *   T'[i][j] = c + k * ( P[i][j] + ((S+N) - 2c)*ry + ((E+W) - 2c)*rx + (amb - c)*rz )
 */
static void hotspot_step(const double* t, const double* p, double* out, long R, long C,
                         double k, double rx, double ry, double rz, double amb) {
    ORACLE_PAR
    for (long i = 0; i < R; ++i) {
        long in = lmax(i - 1, 0), is = lmin(i + 1, R - 1);
        for (long j = 0; j < C; ++j) {
            long jw = lmax(j - 1, 0), je = lmin(j + 1, C - 1);
            double c = t[i * C + j];
            double n = t[in * C + j], s = t[is * C + j];
            double w = t[i * C + jw], e = t[i * C + je];
            double a = (s + n) - 2.0 * c;
            double b = (e + w) - 2.0 * c;
            double d = amb - c;
            double acc = p[i * C + j] + a * ry;
            acc = acc + b * rx;
            acc = acc + d * rz;
            out[i * C + j] = c + k * acc;
        }
    }
}

/* `iters` steps starting from T0; result in out (T0 untouched).  iters == 0 copies T0. */
int oracle_hotspot(const double* t0, const double* p, double* out, long R, long C, int iters,
                   double k, double rx, double ry, double rz, double amb) {
    if (!t0 || !p || !out || R < 1 || C < 1 || iters < 0) return ORACLE_EINVAL;
    size_t n = (size_t)R * (size_t)C;
    double* cur = (double*)malloc(n * sizeof(double));
    double* nxt = (double*)malloc(n * sizeof(double));
    if (!cur || !nxt) { free(cur); free(nxt); return ORACLE_ENOMEM; }
    memcpy(cur, t0, n * sizeof(double));
    for (int it = 0; it < iters; ++it) {
        hotspot_step(cur, p, nxt, R, C, k, rx, ry, rz, amb);
        double* tmp = cur; cur = nxt; nxt = tmp;
    }
    memcpy(out, cur, n * sizeof(double));
    free(cur); free(nxt);
    return ORACLE_OK;
}

/* ------------------------------------------------------------------------------------ */
/* srad_v2 (Rodinia srad_v2 CPU path; readings S1-S9)
 *
 * ROI statistics over rows r1..r2, cols c1..c2 (inclusive), accumulated in fp64:
 *   nR = (r2-r1+1)(c2-c1+1); mean = sum/nR; var = sum2/nR - mean^2; q0sqr = var/mean^2
 */
int oracle_srad_q0sqr(const double* J, long R, long C, long r1, long r2, long c1, long c2,
                      double* q0sqr) {
    if (!J || !q0sqr || R < 1 || C < 1 || r1 < 0 || c1 < 0 || r2 < r1 || c2 < c1 ||
        r2 >= R || c2 >= C)
        return ORACLE_EINVAL;
    double sum = 0.0, sum2 = 0.0;
    for (long i = r1; i <= r2; ++i)
        for (long j = c1; j <= c2; ++j) {
            double v = J[i * C + j];
            sum += v;
            sum2 += v * v;
        }
    double nr = (double)((r2 - r1 + 1) * (c2 - c1 + 1));
    double mean = sum / nr;
    double var = sum2 / nr - mean * mean;
    if (mean == 0.0) return ORACLE_EDEGENERATE;
    *q0sqr = var / (mean * mean);
    return ORACLE_OK;
}

/* Pass 1 (srad_cuda_1): diffusion coefficient of every cell from the OLD image J.
 *   dN = J[max(i-1,0)][j]-Jc, dS = J[min(i+1,R-1)][j]-Jc, dW = J[i][max(j-1,0)]-Jc,
 *   dE = J[i][min(j+1,C-1)]-Jc
 *   G2 = (dN^2+dS^2+dW^2+dE^2)/Jc^2 ; L = (dN+dS+dW+dE)/Jc
 *   num = 0.5*G2 - (1/16)*L^2 ; den = 1 + 0.25*L ; qsqr = num/den^2
 *   t = (qsqr == q0sqr) ? 0 : (qsqr - q0sqr) / (q0sqr*(1+q0sqr))   (reading S3)
 *   c = 1/(1+t), clamped to [0, 1]
 * Writes c (R*C).  The four differences are recomputed by pass 2 from the same J. */
int oracle_srad_coeff(const double* J, long R, long C, double q0sqr, double* cout) {
    if (!J || !cout || R < 1 || C < 1) return ORACLE_EINVAL;
    ORACLE_PAR
    for (long i = 0; i < R; ++i) {
        long in = lmax(i - 1, 0), is = lmin(i + 1, R - 1);
        for (long j = 0; j < C; ++j) {
            long jw = lmax(j - 1, 0), je = lmin(j + 1, C - 1);
            double jc = J[i * C + j];
            double dn = J[in * C + j] - jc, ds = J[is * C + j] - jc;
            double dw = J[i * C + jw] - jc, de = J[i * C + je] - jc;
            double g2 = (dn * dn + ds * ds + dw * dw + de * de) / (jc * jc);
            double l = (dn + ds + dw + de) / jc;
            double num = 0.5 * g2 - (1.0 / 16.0) * (l * l);
            double den = 1.0 + 0.25 * l;
            double qsqr = num / (den * den);
            double t = (qsqr == q0sqr) ? 0.0 : (qsqr - q0sqr) / (q0sqr * (1.0 + q0sqr));
            double c = 1.0 / (1.0 + t);
            if (c < 0.0) c = 0.0;
            else if (c > 1.0) c = 1.0;
            cout[i * C + j] = c;
        }
    }
    return ORACLE_OK;
}

/* Pass 2 (srad_cuda_2), Jacobi: all differences from the OLD J, all c from pass 1.
 *   D = c[i][j]*dN + c[min(i+1,R-1)][j]*dS + c[i][j]*dW + c[i][min(j+1,C-1)]*dE
 *   J'[i][j] = J[i][j] + 0.25*lambda*D
 * jold and jnew must not alias. */
static void srad_update(const double* jold, const double* c, double* jnew, long R, long C,
                        double lambda) {
    ORACLE_PAR
    for (long i = 0; i < R; ++i) {
        long in = lmax(i - 1, 0), is = lmin(i + 1, R - 1);
        for (long j = 0; j < C; ++j) {
            long jw = lmax(j - 1, 0), je = lmin(j + 1, C - 1);
            double jc = jold[i * C + j];
            double dn = jold[in * C + j] - jc, ds = jold[is * C + j] - jc;
            double dw = jold[i * C + jw] - jc, de = jold[i * C + je] - jc;
            double cn = c[i * C + j], cs = c[is * C + j];
            double cw = c[i * C + j], ce = c[i * C + je];
            double d = cn * dn + cs * ds + cw * dw + ce * de;
            jnew[i * C + j] = jc + 0.25 * lambda * d;
        }
    }
}

/* One srad iteration with an externally supplied q0sqr (used by the windowed tests,
 * which take q0sqr(t) from the full-grid ROI). J updated in place. */
int oracle_srad_step(double* J, long R, long C, double q0sqr, double lambda) {
    if (!J || R < 1 || C < 1) return ORACLE_EINVAL;
    size_t n = (size_t)R * (size_t)C;
    double* c = (double*)malloc(n * sizeof(double));
    double* jn = (double*)malloc(n * sizeof(double));
    if (!c || !jn) { free(c); free(jn); return ORACLE_ENOMEM; }
    oracle_srad_coeff(J, R, C, q0sqr, c);
    srad_update(J, c, jn, R, C, lambda);
    memcpy(J, jn, n * sizeof(double));
    free(c); free(jn);
    return ORACLE_OK;
}

/* niter iterations; each starts with the ROI statistics of the current J.
 * q0_seq (nullable, length niter) receives the q0sqr of each iteration. */
int oracle_srad(double* J, long R, long C, long r1, long r2, long c1, long c2, double lambda,
                int niter, double* q0_seq) {
    if (!J || R < 1 || C < 1 || niter < 0 || !isfinite(lambda)) return ORACLE_EINVAL;
    if (r1 < 0 || c1 < 0 || r2 < r1 || c2 < c1 || r2 >= R || c2 >= C) return ORACLE_EINVAL;
    for (int it = 0; it < niter; ++it) {
        double q0;
        int st = oracle_srad_q0sqr(J, R, C, r1, r2, c1, c2, &q0);
        if (st) return st;
        if (q0_seq) q0_seq[it] = q0;
        st = oracle_srad_step(J, R, C, q0, lambda);
        if (st) return st;
    }
    return ORACLE_OK;
}

/* ------------------------------------------------------------------------------------ */
/* pathfinder (Rodinia pathfinder `dynproc_kernel`; readings P1-P6)
 *   prev = wall[0]; for r = 1..R-1:
 *     next[j] = wall[r][j] + min(prev[j-1] (j>0), prev[j], prev[j+1] (j<C-1))
 *   result = prev after the last row. int32 arithmetic (overflow is the caller's contract). */
int oracle_pathfinder(const int32_t* wall, long R, long C, int32_t* result) {
    if (!wall || !result || R < 1 || C < 1) return ORACLE_EINVAL;
    int32_t* prev = (int32_t*)malloc((size_t)C * sizeof(int32_t));
    int32_t* next = (int32_t*)malloc((size_t)C * sizeof(int32_t));
    if (!prev || !next) { free(prev); free(next); return ORACLE_ENOMEM; }
    memcpy(prev, wall, (size_t)C * sizeof(int32_t));
    for (long r = 1; r < R; ++r) {
        ORACLE_PAR
        for (long j = 0; j < C; ++j) {
            int32_t m = prev[j];
            if (j > 0 && prev[j - 1] < m) m = prev[j - 1];
            if (j < C - 1 && prev[j + 1] < m) m = prev[j + 1];
            next[j] = wall[r * C + j] + m;
        }
        int32_t* tmp = prev; prev = next; next = tmp;
    }
    memcpy(result, prev, (size_t)C * sizeof(int32_t));
    free(prev); free(next);
    return ORACLE_OK;
}

/* ------------------------------------------------------------------------------------ */
/* lud (Rodinia lud `lud_base`; readings L1-L6)
 * Doolittle LU without pivoting, packed in place: unit-diagonal L strictly below the
 * diagonal, U on and above it.
 *   U[i][j] = A[i][j] - sum_{k<i} L[i][k] U[k][j]                (j >= i)
 *   L[j][i] = (A[j][i] - sum_{k<i} L[j][k] U[k][i]) / U[i][i]    (j > i)
 * Evaluated row by row (row i is reduced by rows k = 0..i-1 in ascending k), which is
 * the same set of sums in the same k order as the formulas above, with unit stride in j. */
int oracle_lud(double* a, long n) {
    if (!a || n < 1) return ORACLE_EINVAL;
    for (long i = 0; i < n; ++i) {
        double* ri = a + i * n;
        for (long k = 0; k < i; ++k) {
            const double* rk = a + k * n;
            double l = ri[k] / rk[k];
            ri[k] = l;
            for (long j = k + 1; j < n; ++j) ri[j] = ri[j] - l * rk[j];
        }
    }
    return ORACLE_OK;
}

/* ------------------------------------------------------------------------------------ */
/* srad_v1 (Rodinia srad_v1 `extract`, `prepare`+`reduce`, `srad`, `srad2`, `compress`;
 * DESIGN.md readings V1-V4).  The image (pixel values 0..255) is mapped to J = exp(image/255)
 * (extract), niter srad iterations run with the statistics taken over the WHOLE image
 * (srad_v1's ROI is rows 0..R-1, cols 0..C-1), and the result is mapped back with
 * image = log(J)*255 (compress).  The per-iteration arithmetic is srad_v2's (pass 1, pass 2
 * above).  image (R*C) is updated in place. */
int oracle_srad_v1(double* image, long R, long C, double lambda, int niter) {
    if (!image || R < 1 || C < 1 || niter < 0 || !isfinite(lambda)) return ORACLE_EINVAL;
    size_t n = (size_t)R * (size_t)C;
    for (size_t i = 0; i < n; ++i) image[i] = exp(image[i] / 255.0);
    int st = oracle_srad(image, R, C, 0, R - 1, 0, C - 1, lambda, niter, NULL);
    if (st) return st;
    for (size_t i = 0; i < n; ++i) image[i] = log(image[i]) * 255.0;
    return ORACLE_OK;
}

/* ------------------------------------------------------------------------------------ */
/* hotspot3D (Rodinia hotspot3D `hotspotOpt1` / `computeTempCPU`; readings T1-T4).
 * Grid nx (x, fastest) x ny x nz, index c = z*nx*ny + y*nx + x.
 * Chip constants as hotspot; cell sizes dx = chip_h/ny ... Rodinia: dx = chip_height/numRows,
 * dy = chip_width/numCols, dz = t_chip/layers:
 *   Cap = FACTOR_CHIP*SPEC_HEAT_SI*t_chip*dx*dy; Rx = dy/(2 K_SI t_chip dx);
 *   Ry = dx/(2 K_SI t_chip dy); Rz = dz/(K_SI dx dy); dt = PRECISION / (MAX_PD/(FACTOR_CHIP t_chip SPEC_HEAT_SI))
 *   sdc = dt/Cap; ce = cw = sdc/Rx; cn = cs = sdc/Ry; ct = cb = sdc/Rz; cc = 1 - (2ce + 2cn + 3ct)
 * out[0..8] = {cc, cw, ce, cs, cn, cb, ct, sdc, amb}. */
int oracle_hotspot3d_coeffs(long nx, long ny, long nz, double chip_w, double chip_h, double t_chip,
                            double out[9]) {
    if (nx < 1 || ny < 1 || nz < 1 || !(chip_w > 0) || !(chip_h > 0) || !(t_chip > 0) || !out)
        return ORACLE_EINVAL;
    const double k_si = 100.0, spec_heat_si = 1.75e6, factor_chip = 0.5, max_pd = 3.0e6;
    const double precision = 0.001, amb = 80.0;
    double dx = chip_h / (double)ny, dy = chip_w / (double)nx, dz = t_chip / (double)nz;
    double cap = factor_chip * spec_heat_si * t_chip * dx * dy;
    double rx = dy / (2.0 * k_si * t_chip * dx);
    double ry = dx / (2.0 * k_si * t_chip * dy);
    double rz = dz / (k_si * dx * dy);
    double max_slope = max_pd / (factor_chip * t_chip * spec_heat_si);
    double dt = precision / max_slope;
    double sdc = dt / cap;
    double ce = sdc / rx, cn = sdc / ry, ct = sdc / rz;
    out[0] = 1.0 - (2.0 * ce + 2.0 * cn + 3.0 * ct);
    out[1] = ce; out[2] = ce;   /* cw, ce */
    out[3] = cn; out[4] = cn;   /* cs, cn */
    out[5] = ct; out[6] = ct;   /* cb, ct */
    out[7] = sdc;
    out[8] = amb;
    return ORACLE_OK;
}

/* `iters` Jacobi steps of the 7-point stencil, neighbours clamped to the grid:
 *   T' = cc*c + cw*W + ce*E + cs*S + cn*N + cb*B + ct*T + sdc*P + ct*amb
 * (W/E: x-1/x+1, N/S: y-1/y+1, B/T: z-1/z+1), summed left to right. */
int oracle_hotspot3d(const double* t0, const double* p, double* out, long nx, long ny, long nz,
                     int iters, const double cf[9]) {
    if (!t0 || !p || !out || !cf || nx < 1 || ny < 1 || nz < 1 || iters < 0) return ORACLE_EINVAL;
    const double cc = cf[0], cw = cf[1], ce = cf[2], cs = cf[3], cn = cf[4], cb = cf[5], ct = cf[6];
    const double sdc = cf[7], amb = cf[8];
    size_t n = (size_t)nx * ny * nz, plane = (size_t)nx * ny;
    double* cur = (double*)malloc(n * sizeof(double));
    double* nxt = (double*)malloc(n * sizeof(double));
    if (!cur || !nxt) { free(cur); free(nxt); return ORACLE_ENOMEM; }
    memcpy(cur, t0, n * sizeof(double));
    for (int it = 0; it < iters; ++it) {
        ORACLE_PAR
        for (long z = 0; z < nz; ++z)
            for (long y = 0; y < ny; ++y)
                for (long x = 0; x < nx; ++x) {
                    size_t c = (size_t)z * plane + (size_t)y * nx + x;
                    size_t w = x == 0 ? c : c - 1, e = x == nx - 1 ? c : c + 1;
                    size_t nn = y == 0 ? c : c - nx, s = y == ny - 1 ? c : c + nx;
                    size_t b = z == 0 ? c : c - plane, t = z == nz - 1 ? c : c + plane;
                    nxt[c] = cc * cur[c] + cw * cur[w] + ce * cur[e] + cs * cur[s] + cn * cur[nn] +
                             cb * cur[b] + ct * cur[t] + sdc * p[c] + ct * amb;
                }
        double* tmp = cur; cur = nxt; nxt = tmp;
    }
    memcpy(out, cur, n * sizeof(double));
    free(cur); free(nxt);
    return ORACLE_OK;
}

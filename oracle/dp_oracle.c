/*
 * dp_oracle.c — plain fp64 CPU oracle for DREAMPlace's objective/gradient evaluation.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no code, header,
 * table or constant with the CUDA path (paper_conf_dac_lindlrkp19_b200/csrc) and neither
 * side includes or imports the other.
 *
 * Citations: "P:n" = /root/reference/PAPER.md line n (TCAD extension of DAC'19 DREAMPlace).
 * Readings of garbled / silent passages are numbered A1..A26 as in SURVEY.md §8(c) and
 * repeated in DESIGN.md §3.
 *
 * Every function is a direct transcription of a definition, evaluated in double precision,
 * with plain loops.  No blocking, fusion or reordering beyond the definition.  OpenMP is
 * used only where iterations are independent and each output element's arithmetic is
 * unchanged (rows of a transform, cells of the gather), so results are deterministic.
 *
 * Build: gcc -O2 -fopenmp -ffp-contract=off -shared -fPIC dp_oracle.c -lm
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#ifndef M_PI
#define M_PI 3.14159265358979323846
#endif

/* ------------------------------------------------------------------------------------
 * Weighted-average wirelength, one axis of one net.
 *   Table I: x_e^+ = max x_i, x_e^- = min x_i,
 *     a_i^+ = exp((x_i - x_e^+)/gamma),  a_i^- = exp(-(x_i - x_e^-)/gamma)   (P:159 shift)
 *     b_e^+- = sum a_i^+-,  c_e^+- = sum x_i a_i^+-
 *   eq (3) with the shift of P:159:  WL_e = c^+/b^+ - c^-/b^-
 *   eq (6):
 *     dWL_e/dx_i = ((1 + x_i/gamma) b^+ - c^+/gamma)/(b^+)^2 * a_i^+
 *                - ((1 - x_i/gamma) b^- + c^-/gamma)/(b^-)^2 * a_i^-
 *   Nets of degree 0 or 1 contribute WL = 0 and gradient 0 (reading A3).
 * p[i] are the pin coordinates of the net, a_p / a_m are caller scratch of length d.
 * ---------------------------------------------------------------------------------- */
static double wa_axis(int d, const double *p, double gamma, double *grad, double *a_p, double *a_m)
{
    if (d < 2) {
        for (int i = 0; i < d; i++) grad[i] = 0.0;
        return 0.0;
    }
    double xp = p[0], xm = p[0];
    for (int i = 1; i < d; i++) {
        if (p[i] > xp) xp = p[i];
        if (p[i] < xm) xm = p[i];
    }
    double bp = 0.0, bm = 0.0, cp = 0.0, cm = 0.0;
    for (int i = 0; i < d; i++) {
        a_p[i] = exp((p[i] - xp) / gamma);
        a_m[i] = exp(-(p[i] - xm) / gamma);
        bp += a_p[i];
        bm += a_m[i];
        cp += p[i] * a_p[i];
        cm += p[i] * a_m[i];
    }
    double wl = cp / bp - cm / bm;
    for (int i = 0; i < d; i++) {
        double gp = ((1.0 + p[i] / gamma) * bp - cp / gamma) / (bp * bp) * a_p[i];
        double gm = ((1.0 - p[i] / gamma) * bm + cm / gamma) / (bm * bm) * a_m[i];
        grad[i] = gp - gm;
    }
    return wl;
}

/* Sum over nets of w_e (WL_e^x + WL_e^y)  (eq 2's first term), and the cell gradient:
 * pin location px = x[cell] + dx (reading A1: x is the cell's lower-left corner, offsets are
 * relative to it); a cell's gradient is the sum of its pins' gradients.
 * gx, gy (length num_cells) are accumulated into (caller zeroes them).
 * wl_net (nullable) receives w_e (WL_e^x + WL_e^y) per net.  Returns the total. */
double or_wa(int64_t num_nets, const int32_t *net_start, const int32_t *pin2cell,
             const double *pin_dx, const double *pin_dy, const double *net_weight,
             const double *x, const double *y, double gamma,
             double *gx, double *gy, double *wl_net)
{
    int dmax = 0;
    for (int64_t e = 0; e < num_nets; e++) {
        int d = net_start[e + 1] - net_start[e];
        if (d > dmax) dmax = d;
    }
    size_t n = (size_t)(dmax > 0 ? dmax : 1);
    double *px = malloc(n * sizeof(double)), *py = malloc(n * sizeof(double));
    double *gxp = malloc(n * sizeof(double)), *gyp = malloc(n * sizeof(double));
    double *ap = malloc(n * sizeof(double)), *am = malloc(n * sizeof(double));
    double total = 0.0;
    for (int64_t e = 0; e < num_nets; e++) {
        int s = net_start[e], d = net_start[e + 1] - s;
        for (int i = 0; i < d; i++) {
            int c = pin2cell[s + i];
            px[i] = x[c] + pin_dx[s + i];
            py[i] = y[c] + pin_dy[s + i];
        }
        double we = net_weight ? net_weight[e] : 1.0;
        double wlx = wa_axis(d, px, gamma, gxp, ap, am);
        double wly = wa_axis(d, py, gamma, gyp, ap, am);
        double wl = we * (wlx + wly);
        if (wl_net) wl_net[e] = wl;
        total += wl;
        for (int i = 0; i < d; i++) {
            int c = pin2cell[s + i];
            gx[c] += we * gxp[i];
            gy[c] += we * gyp[i];
        }
    }
    free(px); free(py); free(gxp); free(gyp); free(ap); free(am);
    return total;
}

/* ------------------------------------------------------------------------------------
 * Log-sum-exp wirelength, one axis of one net (NEXT-3; "log-sum-exp (LSE) [29], which is
 * also implemented in the framework").  The paper prints no LSE formula; reading A27
 * takes the standard definition of [29] (Naylor et al.):
 *   LSE_e = gamma ln sum_i exp(x_i/gamma) + gamma ln sum_i exp(-x_i/gamma)
 * evaluated with the same overflow-safe shift as WA and Table I's a_i^+-, b_e^+-:
 *   LSE_e = (x_e^+ + gamma ln b_e^+) - (x_e^- - gamma ln b_e^-)
 *   dLSE_e/dx_i = a_i^+/b_e^+ - a_i^-/b_e^-
 * Nets of degree 0 or 1 contribute 0 (reading A3).
 * ---------------------------------------------------------------------------------- */
static double lse_axis(int d, const double *p, double gamma, double *grad, double *a_p, double *a_m)
{
    if (d < 2) {
        for (int i = 0; i < d; i++) grad[i] = 0.0;
        return 0.0;
    }
    double xp = p[0], xm = p[0];
    for (int i = 1; i < d; i++) {
        if (p[i] > xp) xp = p[i];
        if (p[i] < xm) xm = p[i];
    }
    double bp = 0.0, bm = 0.0;
    for (int i = 0; i < d; i++) {
        a_p[i] = exp((p[i] - xp) / gamma);
        a_m[i] = exp(-(p[i] - xm) / gamma);
        bp += a_p[i];
        bm += a_m[i];
    }
    double wl = (xp + gamma * log(bp)) - (xm - gamma * log(bm));
    for (int i = 0; i < d; i++) grad[i] = a_p[i] / bp - a_m[i] / bm;
    return wl;
}

/* Sum over nets of w_e (LSE_e^x + LSE_e^y) and its cell gradient, with the same pin model
 * (reading A1) and accumulation contract as or_wa. */
double or_lse(int64_t num_nets, const int32_t *net_start, const int32_t *pin2cell,
              const double *pin_dx, const double *pin_dy, const double *net_weight,
              const double *x, const double *y, double gamma,
              double *gx, double *gy, double *wl_net)
{
    int dmax = 0;
    for (int64_t e = 0; e < num_nets; e++) {
        int d = net_start[e + 1] - net_start[e];
        if (d > dmax) dmax = d;
    }
    size_t n = (size_t)(dmax > 0 ? dmax : 1);
    double *px = malloc(n * sizeof(double)), *py = malloc(n * sizeof(double));
    double *gxp = malloc(n * sizeof(double)), *gyp = malloc(n * sizeof(double));
    double *ap = malloc(n * sizeof(double)), *am = malloc(n * sizeof(double));
    double total = 0.0;
    for (int64_t e = 0; e < num_nets; e++) {
        int s = net_start[e], d = net_start[e + 1] - s;
        for (int i = 0; i < d; i++) {
            int c = pin2cell[s + i];
            px[i] = x[c] + pin_dx[s + i];
            py[i] = y[c] + pin_dy[s + i];
        }
        double we = net_weight ? net_weight[e] : 1.0;
        double wl = we * (lse_axis(d, px, gamma, gxp, ap, am) + lse_axis(d, py, gamma, gyp, ap, am));
        if (wl_net) wl_net[e] = wl;
        total += wl;
        for (int i = 0; i < d; i++) {
            int c = pin2cell[s + i];
            gx[c] += we * gxp[i];
            gy[c] += we * gyp[i];
        }
    }
    free(px); free(py); free(gxp); free(gyp); free(ap); free(am);
    return total;
}

/* Per-net half-perimeter wirelength (named at P:95, used by eq 18's p at P:450; reading A6):
 *   h_e = (max px - min px) + (max py - min py),  px = x[cell] + dx in fp64;  d <= 1 -> 0.
 * The correctly rounded total is formed by the caller (math.fsum, reading A7). */
void or_hpwl_nets(int64_t num_nets, const int32_t *net_start, const int32_t *pin2cell,
                  const double *pin_dx, const double *pin_dy, const double *x, const double *y,
                  double *h_net)
{
    for (int64_t e = 0; e < num_nets; e++) {
        int s = net_start[e], d = net_start[e + 1] - s;
        if (d < 2) { h_net[e] = 0.0; continue; }
        double xp = -INFINITY, xm = INFINITY, yp = -INFINITY, ym = INFINITY;
        for (int i = 0; i < d; i++) {
            int c = pin2cell[s + i];
            double px = x[c] + pin_dx[s + i], py = y[c] + pin_dy[s + i];
            if (px > xp) xp = px;
            if (px < xm) xm = px;
            if (py > yp) yp = py;
            if (py < ym) ym = py;
        }
        h_net[e] = (xp - xm) + (yp - ym);
    }
}

/* ------------------------------------------------------------------------------------
 * Cell footprint on the bin grid (density map P:253; force P:320).
 * Reading A10 (stretch): w' = max(w, sqrt2*bx), h' = max(h, sqrt2*by), box centred on the
 * cell centre (x + w/2, y + h/2), charge scaled by r = w h / (w' h').  stretch = 0 gives
 * the literal overlap (w' = w, r = 1).  Reading A11: overlap is clipped to the region.
 * ---------------------------------------------------------------------------------- */
typedef struct { double lo_x, hi_x, lo_y, hi_y, r; } footprint;

static footprint cell_footprint(double x, double y, double w, double h,
                                double xl, double yl, double xh, double yh,
                                double bx, double by, int stretch)
{
    footprint f;
    double ws = w, hs = h;
    if (stretch) {
        double sx = sqrt(2.0) * bx, sy = sqrt(2.0) * by;
        if (ws < sx) ws = sx;
        if (hs < sy) hs = sy;
    }
    f.r = (ws * hs > 0.0) ? (w * h) / (ws * hs) : 0.0;
    double cx = x + 0.5 * w, cy = y + 0.5 * h;
    f.lo_x = cx - 0.5 * ws; f.hi_x = cx + 0.5 * ws;
    f.lo_y = cy - 0.5 * hs; f.hi_y = cy + 0.5 * hs;
    if (f.lo_x < xl) f.lo_x = xl;
    if (f.hi_x > xh) f.hi_x = xh;
    if (f.lo_y < yl) f.lo_y = yl;
    if (f.hi_y > yh) f.hi_y = yh;
    return f;
}

/* overlap length of [lo, hi] with bin i = [o + i b, o + (i+1) b] */
static double overlap_1d(double lo, double hi, double o, double b, int i)
{
    double a = o + i * b, c = o + (i + 1) * b;
    double l = lo > a ? lo : a, u = hi < c ? hi : c;
    return u > l ? u - l : 0.0;
}

static void bin_range(double lo, double hi, double o, double b, int m, int *i0, int *i1)
{
    int a = (int)floor((lo - o) / b), c = (int)floor((hi - o) / b);
    if (a < 0) a = 0;
    if (c > m - 1) c = m - 1;
    *i0 = a; *i1 = c;
}

/* Density map rho[bx][by] (row-major, y contiguous; reading A20), dimensionless
 * (reading A9):  rho_b = sum_i r_i ovx_i(bx) ovy_i(by) / (bin_w bin_h).
 * rho must be zeroed by the caller. */
void or_density_map(int64_t num_cells, const double *x, const double *y,
                    const double *w, const double *h,
                    double xl, double yl, double xh, double yh, int mx, int my, int stretch,
                    double *rho)
{
    double bx = (xh - xl) / mx, by = (yh - yl) / my;
    for (int64_t c = 0; c < num_cells; c++) {
        footprint f = cell_footprint(x[c], y[c], w[c], h[c], xl, yl, xh, yh, bx, by, stretch);
        if (f.hi_x <= f.lo_x || f.hi_y <= f.lo_y || f.r == 0.0) continue;
        int i0, i1, j0, j1;
        bin_range(f.lo_x, f.hi_x, xl, bx, mx, &i0, &i1);
        bin_range(f.lo_y, f.hi_y, yl, by, my, &j0, &j1);
        for (int i = i0; i <= i1; i++) {
            double ox = overlap_1d(f.lo_x, f.hi_x, xl, bx, i);
            if (ox <= 0.0) continue;
            for (int j = j0; j <= j1; j++) {
                double oy = overlap_1d(f.lo_y, f.hi_y, yl, by, j);
                if (oy <= 0.0) continue;
                rho[(int64_t)i * my + j] += f.r * ox * oy / (bx * by);
            }
        }
    }
}

/* Electric force on each cell: the force is the sum over overlapped bins of
 * overlap area x field; the density gradient is its negative (reading A21):
 *   dD/dx_i = - sum_b r_i ov(i,b) xi^X_b,   dD/dy_i = - sum_b r_i ov(i,b) xi^Y_b
 * Footprint identical to or_density_map.  gx, gy are overwritten. */
void or_density_grad(int64_t num_cells, const double *x, const double *y,
                     const double *w, const double *h,
                     double xl, double yl, double xh, double yh, int mx, int my, int stretch,
                     const double *xi_x, const double *xi_y, double *gx, double *gy)
{
    double bx = (xh - xl) / mx, by = (yh - yl) / my;
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t c = 0; c < num_cells; c++) {
        footprint f = cell_footprint(x[c], y[c], w[c], h[c], xl, yl, xh, yh, bx, by, stretch);
        double sx = 0.0, sy = 0.0;
        if (f.hi_x > f.lo_x && f.hi_y > f.lo_y && f.r != 0.0) {
            int i0, i1, j0, j1;
            bin_range(f.lo_x, f.hi_x, xl, bx, mx, &i0, &i1);
            bin_range(f.lo_y, f.hi_y, yl, by, my, &j0, &j1);
            for (int i = i0; i <= i1; i++) {
                double ox = overlap_1d(f.lo_x, f.hi_x, xl, bx, i);
                if (ox <= 0.0) continue;
                for (int j = j0; j <= j1; j++) {
                    double oy = overlap_1d(f.lo_y, f.hi_y, yl, by, j);
                    if (oy <= 0.0) continue;
                    double ov = f.r * ox * oy;
                    sx += ov * xi_x[(int64_t)i * my + j];
                    sy += ov * xi_y[(int64_t)i * my + j];
                }
            }
        }
        gx[c] = -sx;
        gy[c] = -sy;
    }
}

/* ------------------------------------------------------------------------------------
 * 1-D transforms along the last (contiguous) axis of a rows x n array, naive O(n^2):
 *   kind 0  DCT,   eq (7a) scaled by 2/n (reading A13: the normalisation of
 *           Alg 3 line 12, so that IDCT(DCT(x)) = x):
 *             out_k = (2/n) sum_{t=0}^{n-1} x_t cos(pi/n (t + 1/2) k)
 *   kind 1  IDCT,  eq (7b):  out_k = x_0/2 + sum_{t=1}^{n-1} x_t cos(pi/n t (k + 1/2))
 *   kind 2  IDXST, eq (8a):  out_k = sum_{t=0}^{n-1} x_t sin(pi/n t (k + 1/2))
 * The integer phase is reduced mod 4n before calling cos/sin (exact integer arithmetic);
 * angle = pi * m / (2n) with m = (2t+1)k or t(2k+1).
 * ---------------------------------------------------------------------------------- */
void or_transform_lastaxis(int kind, int64_t rows, int n, const double *in, double *out)
{
    double *tab = malloc((size_t)n * n * sizeof(double));
    for (int k = 0; k < n; k++) {
        for (int t = 0; t < n; t++) {
            int64_t m = (kind == 0) ? (int64_t)(2 * t + 1) * k : (int64_t)t * (2 * k + 1);
            m %= 4LL * n;
            double ang = M_PI * (double)m / (2.0 * n);
            tab[(size_t)k * n + t] = (kind == 2) ? sin(ang) : cos(ang);
        }
    }
#pragma omp parallel for schedule(static)
    for (int64_t r = 0; r < rows; r++) {
        const double *src = in + r * n;
        double *dst = out + r * n;
        for (int k = 0; k < n; k++) {
            const double *tk = tab + (size_t)k * n;
            double s;
            if (kind == 0) {
                s = 0.0;
                for (int t = 0; t < n; t++) s += src[t] * tk[t];
                s *= 2.0 / n;
            } else if (kind == 1) {
                s = 0.5 * src[0];
                for (int t = 1; t < n; t++) s += src[t] * tk[t];
            } else {
                s = 0.0;
                for (int t = 0; t < n; t++) s += src[t] * tk[t];
            }
            dst[k] = s;
        }
    }
    free(tab);
}


/* ====================================================================================
 * TIMED MODE (the CPU baseline of BASELINE.md §4; never used for parity).
 * The same definitions as above, organised for speed the way the paper's CPU version runs
 * them: OpenMP over nets and over cells with dynamic scheduling and the paper's chunk sizes
 * |E| / (T 16) and |V| / (T 16), atomic accumulation of the cell gradient and
 * of the bin map, and the 1-D transforms by a textbook fp64 N-point FFT in Makhoul's order
 * (Alg 3) instead of the naive O(N^2) sums.  tests/test_oracle_timed.py checks
 * every function here against the plain functions above.
 * ==================================================================================== */
#include <omp.h>

static int64_t chunk_of(int64_t n, int threads)
{
    int64_t c = n / ((int64_t)threads * 16);
    return c > 0 ? c : 1;
}

double or_wa_omp(int threads, int64_t num_nets, const int32_t *net_start, const int32_t *pin2cell,
                 const double *pin_dx, const double *pin_dy, const double *net_weight,
                 const double *x, const double *y, double gamma, double *gx, double *gy)
{
    int dmax = 1;
    for (int64_t e = 0; e < num_nets; e++) {
        int d = net_start[e + 1] - net_start[e];
        if (d > dmax) dmax = d;
    }
    const int64_t chunk = chunk_of(num_nets, threads);
    double total = 0.0;
#pragma omp parallel num_threads(threads) reduction(+ : total)
    {
        size_t n = (size_t)dmax;
        double *px = malloc(n * sizeof(double)), *py = malloc(n * sizeof(double));
        double *gxp = malloc(n * sizeof(double)), *gyp = malloc(n * sizeof(double));
        double *ap = malloc(n * sizeof(double)), *am = malloc(n * sizeof(double));
#pragma omp for schedule(dynamic, chunk)
        for (int64_t e = 0; e < num_nets; e++) {
            int s = net_start[e], d = net_start[e + 1] - s;
            for (int i = 0; i < d; i++) {
                int c = pin2cell[s + i];
                px[i] = x[c] + pin_dx[s + i];
                py[i] = y[c] + pin_dy[s + i];
            }
            double we = net_weight ? net_weight[e] : 1.0;
            total += we * (wa_axis(d, px, gamma, gxp, ap, am) + wa_axis(d, py, gamma, gyp, ap, am));
            for (int i = 0; i < d; i++) {
                int c = pin2cell[s + i];
#pragma omp atomic
                gx[c] += we * gxp[i];
#pragma omp atomic
                gy[c] += we * gyp[i];
            }
        }
        free(px); free(py); free(gxp); free(gyp); free(ap); free(am);
    }
    return total;
}

void or_density_map_omp(int threads, int64_t num_cells, const double *x, const double *y,
                        const double *w, const double *h, double xl, double yl, double xh, double yh,
                        int mx, int my, int stretch, double *rho)
{
    double bx = (xh - xl) / mx, by = (yh - yl) / my;
    const int64_t chunk = chunk_of(num_cells, threads);
#pragma omp parallel for num_threads(threads) schedule(dynamic, chunk)
    for (int64_t c = 0; c < num_cells; c++) {
        footprint f = cell_footprint(x[c], y[c], w[c], h[c], xl, yl, xh, yh, bx, by, stretch);
        if (f.hi_x <= f.lo_x || f.hi_y <= f.lo_y || f.r == 0.0) continue;
        int i0, i1, j0, j1;
        bin_range(f.lo_x, f.hi_x, xl, bx, mx, &i0, &i1);
        bin_range(f.lo_y, f.hi_y, yl, by, my, &j0, &j1);
        for (int i = i0; i <= i1; i++) {
            double ox = overlap_1d(f.lo_x, f.hi_x, xl, bx, i);
            if (ox <= 0.0) continue;
            for (int j = j0; j <= j1; j++) {
                double oy = overlap_1d(f.lo_y, f.hi_y, yl, by, j);
                if (oy <= 0.0) continue;
#pragma omp atomic
                rho[(int64_t)i * my + j] += f.r * ox * oy / (bx * by);
            }
        }
    }
}

void or_density_grad_omp(int threads, int64_t num_cells, const double *x, const double *y,
                         const double *w, const double *h, double xl, double yl, double xh, double yh,
                         int mx, int my, int stretch, const double *xi_x, const double *xi_y,
                         double *gx, double *gy)
{
    double bx = (xh - xl) / mx, by = (yh - yl) / my;
    const int64_t chunk = chunk_of(num_cells, threads);
#pragma omp parallel for num_threads(threads) schedule(dynamic, chunk)
    for (int64_t c = 0; c < num_cells; c++) {
        footprint f = cell_footprint(x[c], y[c], w[c], h[c], xl, yl, xh, yh, bx, by, stretch);
        double sx = 0.0, sy = 0.0;
        if (f.hi_x > f.lo_x && f.hi_y > f.lo_y && f.r != 0.0) {
            int i0, i1, j0, j1;
            bin_range(f.lo_x, f.hi_x, xl, bx, mx, &i0, &i1);
            bin_range(f.lo_y, f.hi_y, yl, by, my, &j0, &j1);
            for (int i = i0; i <= i1; i++) {
                double ox = overlap_1d(f.lo_x, f.hi_x, xl, bx, i);
                if (ox <= 0.0) continue;
                for (int j = j0; j <= j1; j++) {
                    double oy = overlap_1d(f.lo_y, f.hi_y, yl, by, j);
                    if (oy <= 0.0) continue;
                    double ov = f.r * ox * oy;
                    sx += ov * xi_x[(int64_t)i * my + j];
                    sy += ov * xi_y[(int64_t)i * my + j];
                }
            }
        }
        gx[c] = -sx;
        gy[c] = -sy;
    }
}

/* In-place iterative radix-2 complex FFT (textbook Cooley-Tukey, bit-reversal first),
 * n a power of two; sign = -1: X_k = sum_m v_m e^{-2 pi i k m / n}, +1: the unnormalised
 * inverse.  re/im hold the sequence; tc/ts = cos/sin(2 pi k / n), k < n/2. */
static void fft_inplace(int n, double *re, double *im, const double *tc, const double *ts, int sign)
{
    for (int i = 1, j = 0; i < n; i++) {
        int bit = n >> 1;
        for (; j & bit; bit >>= 1) j ^= bit;
        j ^= bit;
        if (i < j) {
            double t = re[i]; re[i] = re[j]; re[j] = t;
            t = im[i]; im[i] = im[j]; im[j] = t;
        }
    }
    for (int len = 2; len <= n; len <<= 1) {
        int step = n / len;
        for (int i = 0; i < n; i += len) {
            for (int k = 0; k < len / 2; k++) {
                double wr = tc[k * step], wi = sign * ts[k * step];
                double ur = re[i + k], ui = im[i + k];
                double vr = re[i + k + len / 2] * wr - im[i + k + len / 2] * wi;
                double vi = re[i + k + len / 2] * wi + im[i + k + len / 2] * wr;
                re[i + k] = ur + vr; im[i + k] = ui + vi;
                re[i + k + len / 2] = ur - vr; im[i + k + len / 2] = ui - vi;
            }
        }
    }
}

/* The transforms of or_transform_lastaxis (kinds 0 DCT x 2/n, 1 IDCT eq 7b, 2 IDXST eq 8a)
 * through one n-point complex FFT per row (n a power of two):
 *   DCT   (Makhoul): v_m = x_2m, v_{n-1-m} = x_{2m+1}; out_k = (2/n) Re(e^{-i pi k / 2n} V_k)
 *   IDCT  (the inverse of the same): V_k = e^{+i pi k / 2n} (X_k - i X_{n-k}), X_n := 0;
 *         v = unnormalised inverse FFT of V; out_{2m} = Re v_m / 2, out_{2m+1} = Re v_{n-1-m} / 2
 *   IDXST by eq (8e): out_k = (-1)^k IDCT(x')_k with x'_t = x_{n-t}, x'_0 = 0. */
void or_transform_fft(int threads, int kind, int64_t rows, int n, const double *in, double *out)
{
    double *tc = malloc((size_t)(n / 2 > 0 ? n / 2 : 1) * sizeof(double));
    double *ts = malloc((size_t)(n / 2 > 0 ? n / 2 : 1) * sizeof(double));
    for (int k = 0; k < n / 2; k++) {
        tc[k] = cos(2.0 * M_PI * k / n);
        ts[k] = -sin(2.0 * M_PI * k / n);   /* forward twiddle e^{-2 pi i k / n} */
    }
#pragma omp parallel num_threads(threads)
    {
        double *re = malloc((size_t)n * sizeof(double)), *im = malloc((size_t)n * sizeof(double));
        double *xs = malloc((size_t)n * sizeof(double));
#pragma omp for schedule(static)
        for (int64_t r = 0; r < rows; r++) {
            const double *src = in + r * n;
            double *dst = out + r * n;
            if (kind == 0) {
                for (int m = 0; m < n / 2; m++) {
                    re[m] = src[2 * m];
                    re[n - 1 - m] = src[2 * m + 1];
                }
                for (int m = 0; m < n; m++) im[m] = 0.0;
                fft_inplace(n, re, im, tc, ts, 1);
                for (int k = 0; k < n; k++) {
                    double a = M_PI * k / (2.0 * n);
                    dst[k] = (2.0 / n) * (re[k] * cos(a) + im[k] * sin(a));
                }
            } else {
                if (kind == 2) {   /* eq (8e): x'_t = x_{n-t}, x'_0 = 0 */
                    xs[0] = 0.0;
                    for (int t = 1; t < n; t++) xs[t] = src[n - t];
                } else {
                    memcpy(xs, src, (size_t)n * sizeof(double));
                }
                for (int k = 0; k < n; k++) {
                    double xr = xs[k], xi = (k == 0) ? 0.0 : -xs[n - k];
                    double a = M_PI * k / (2.0 * n), c = cos(a), s = sin(a);
                    re[k] = xr * c - xi * s;
                    im[k] = xr * s + xi * c;
                }
                fft_inplace(n, re, im, tc, ts, -1);
                for (int m = 0; m < n / 2; m++) {
                    dst[2 * m] = 0.5 * re[m];
                    dst[2 * m + 1] = 0.5 * re[n - 1 - m];
                }
                if (kind == 2)
                    for (int k = 1; k < n; k += 2) dst[k] = -dst[k];
            }
        }
        free(re); free(im); free(xs);
    }
    free(tc); free(ts);
}

int or_abi_version(void) { return 1; }

/*
 * ncc_oracle.c -- plain, slow, obviously-correct fp64 CPU oracle for spatial-domain
 * normalized cross-correlation (template matching, TM) and PIV.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_conf_ipps_moorelk13_b200/) never links, imports or calls it, and this file
 * shares no code, header, table or constant generator with the CUDA path.
 *
 * Citations are to /root/reference/PAPER.md as "P:<lines>" plus the figure/section
 * they fall in, and to SURVEY.md section 8(c) ("S8c") where the paper's text is lost.
 *
 * Definition followed (TM, one offset):  MATLAB corr2(template, window)  (Listing 5.1
 * caption P:250-251; Tab 5.1 caption "number of corr2() calls" P:190-191), i.e. the
 * Pearson correlation coefficient with A-bar and B-bar the matrix averages
 * (Fig 5.1 caption P:132-137):
 *
 *     r = sum (A - Abar)(B - Bbar) / sqrt( sum (A - Abar)^2 * sum (B - Bbar)^2 )
 *
 * computed in the two-pass centred form (means first, then centred sums), fp64,
 * serial row-major sums, no blocking or reordering.  Flat template/window
 * (corr2 would give 0/0) -> 0 (S8c reading 4).  Valid offsets only (S8c reading 3).
 *
 * PIV (Figs 5.8-5.12 captions P:164-171; S8c "PIV step by step"): for each window the
 * template is A[y:y+h, x:x+w] and the candidate windows are B[y+dy:.., x+dx:..] for
 * dy in [-my,my], dx in [-mx,mx]; peak = argmax (tie -> smallest row-major index);
 * 3-point Gaussian sub-pixel fit per axis with parabolic fallback (S8c reading 10).
 *
 * Build: gcc -O2 -fopenmp -ffp-contract=off -shared -fPIC ncc_oracle.c -lm
 */
#include <math.h>
#include <stddef.h>
#include <stdint.h>

/* Output flag bits.  Interface values (the same numbers are documented in
 * include/ncc.h and DESIGN.md); restated here so the oracle needs no product header. */
#define OF_FLAT_TEMPLATE 1u
#define OF_EDGE_Y 2u
#define OF_EDGE_X 4u
#define OF_PARABOLA_Y 8u
#define OF_PARABOLA_X 16u
#define OF_INVALID 32u

#define FLAT_REL 1e-10 /* S8c reading 4: relative threshold on fp64 energies */

/* ---------------------------------------------------------------------------
 * corr2 of an h x w template against the h x w window whose top-left corner is
 * img[r0*pitch + c0].  Two-pass centred Pearson, Fig 5.1.
 * ------------------------------------------------------------------------- */
static double corr2_window(const float *img, int64_t pitch, int r0, int c0,
                           const float *tmpl, int64_t tpitch, int h, int w)
{
    const double n = (double)h * (double)w;
    double sumT = 0.0, sumW = 0.0, sumT2 = 0.0, sumW2 = 0.0;
    for (int i = 0; i < h; ++i)
        for (int j = 0; j < w; ++j) {
            double t = tmpl[(int64_t)i * tpitch + j];
            double b = img[(int64_t)(r0 + i) * pitch + (c0 + j)];
            sumT += t;
            sumW += b;
            sumT2 += t * t;
            sumW2 += b * b;
        }
    const double Tbar = sumT / n; /* A-bar: matrix average of the template */
    const double Wbar = sumW / n; /* B-bar: matrix average of the window  */
    double num = 0.0, st = 0.0, sw = 0.0;
    for (int i = 0; i < h; ++i)
        for (int j = 0; j < w; ++j) {
            double a = (double)tmpl[(int64_t)i * tpitch + j] - Tbar;
            double b = (double)img[(int64_t)(r0 + i) * pitch + (c0 + j)] - Wbar;
            num += a * b;
            st += a * a;
            sw += b * b;
        }
    if (st <= FLAT_REL * sumT2 || sw <= FLAT_REL * sumW2)
        return 0.0; /* flat template or flat window: corr2's 0/0 read as 0 (S8c #4) */
    return num / sqrt(st * sw);
}

/* Sum of squared differences of the template against one window: the paper's own PIV
 * similarity score (Fig 5.10 caption: "the per-mask offset sum of squared
 * differences similarity score").  Plain definition, fp64, row-major serial sum. */
static double ssd_window(const float *img, int64_t pitch, int r0, int c0,
                         const float *tmpl, int64_t tpitch, int h, int w)
{
    double s = 0.0;
    for (int i = 0; i < h; ++i)
        for (int j = 0; j < w; ++j) {
            double d = (double)tmpl[(int64_t)i * tpitch + j] -
                       (double)img[(int64_t)(r0 + i) * pitch + (c0 + j)];
            s += d * d;
        }
    return s;
}

/* Sum of absolute differences of the template against one window: the specialisation example
 * of the paper's Ch. 4 ("sum of absolute differences to sum of squared differences")
 * -- the other classic block-matching score.  Plain definition, fp64, row-major serial sum. */
static double sad_window(const float *img, int64_t pitch, int r0, int c0,
                         const float *tmpl, int64_t tpitch, int h, int w)
{
    double s = 0.0;
    for (int i = 0; i < h; ++i)
        for (int j = 0; j < w; ++j)
            s += fabs((double)tmpl[(int64_t)i * tpitch + j] - (double)img[(int64_t)(r0 + i) * pitch + (c0 + j)]);
    return s;
}

/* SAD surface for offset rows [u_begin, u_end) (valid offsets, as oracle_ncc_surface). */
int oracle_sad_surface(const float *img, int H, int W, int64_t pitch,
                       const float *tmpl, int h, int w, int64_t tpitch,
                       int u_begin, int u_end, double *scores)
{
    if (h <= 0 || w <= 0 || h > H || w > W) return -1;
    const int U = H - h + 1, V = W - w + 1;
    if (u_begin < 0 || u_end > U || u_begin > u_end) return -1;
#pragma omp parallel for schedule(dynamic, 1)
    for (int u = u_begin; u < u_end; ++u)
        for (int v = 0; v < V; ++v)
            scores[(int64_t)(u - u_begin) * V + v] = sad_window(img, pitch, u, v, tmpl, tpitch, h, w);
    return 0;
}

/* SSD surface for offset rows [u_begin, u_end) (valid offsets, as oracle_ncc_surface). */
int oracle_ssd_surface(const float *img, int H, int W, int64_t pitch,
                       const float *tmpl, int h, int w, int64_t tpitch,
                       int u_begin, int u_end, double *scores)
{
    if (h <= 0 || w <= 0 || h > H || w > W) return -1;
    const int U = H - h + 1, V = W - w + 1;
    if (u_begin < 0 || u_end > U || u_begin > u_end) return -1;
#pragma omp parallel for schedule(dynamic, 1)
    for (int u = u_begin; u < u_end; ++u)
        for (int v = 0; v < V; ++v)
            scores[(int64_t)(u - u_begin) * V + v] = ssd_window(img, pitch, u, v, tmpl, tpitch, h, w);
    return 0;
}

/* Peak of an SSD surface: argmin, ties -> smallest linear index. */
int64_t oracle_argmin(const double *scores, int64_t count)
{
    int64_t best = 0;
    for (int64_t k = 1; k < count; ++k)
        if (scores[k] < scores[best]) best = k;
    return best;
}

/* Is the template flat?  (S8c reading 4; same energy test as corr2_window.) */
int oracle_template_is_flat(const float *tmpl, int64_t tpitch, int h, int w)
{
    const double n = (double)h * (double)w;
    double s = 0.0, s2 = 0.0;
    for (int i = 0; i < h; ++i)
        for (int j = 0; j < w; ++j) {
            double t = tmpl[(int64_t)i * tpitch + j];
            s += t;
            s2 += t * t;
        }
    const double mean = s / n;
    double st = 0.0;
    for (int i = 0; i < h; ++i)
        for (int j = 0; j < w; ++j) {
            double a = (double)tmpl[(int64_t)i * tpitch + j] - mean;
            st += a * a;
        }
    return st <= FLAT_REL * s2;
}

/* Full TM surface for offset rows [u_begin, u_end): scores[(u-u_begin)*V + v].
 * U = H-h+1, V = W-w+1 (valid offsets only, S8c reading 3). */
int oracle_ncc_surface(const float *img, int H, int W, int64_t pitch,
                       const float *tmpl, int h, int w, int64_t tpitch,
                       int u_begin, int u_end, double *scores)
{
    if (h <= 0 || w <= 0 || h > H || w > W) return -1;
    const int U = H - h + 1, V = W - w + 1;
    if (u_begin < 0 || u_end > U || u_begin > u_end) return -1;
#pragma omp parallel for schedule(dynamic, 1)
    for (int u = u_begin; u < u_end; ++u)
        for (int v = 0; v < V; ++v)
            scores[(int64_t)(u - u_begin) * V + v] =
                corr2_window(img, pitch, u, v, tmpl, tpitch, h, w);
    return 0;
}

/* Scores at an explicit list of offsets (sampled parity at full size). */
int oracle_ncc_at(const float *img, int H, int W, int64_t pitch,
                  const float *tmpl, int h, int w, int64_t tpitch,
                  const int *us, const int *vs, int count, double *out)
{
    if (h <= 0 || w <= 0 || h > H || w > W) return -1;
    const int U = H - h + 1, V = W - w + 1;
    for (int k = 0; k < count; ++k)
        if (us[k] < 0 || us[k] >= U || vs[k] < 0 || vs[k] >= V) return -1;
#pragma omp parallel for schedule(dynamic, 4)
    for (int k = 0; k < count; ++k)
        out[k] = corr2_window(img, pitch, us[k], vs[k], tmpl, tpitch, h, w);
    return 0;
}

/* Peak search over a score array: argmax, ties -> smallest linear index (S8c #5). */
int64_t oracle_argmax(const double *scores, int64_t count)
{
    int64_t best = 0;
    for (int64_t k = 1; k < count; ++k)
        if (scores[k] > scores[best]) best = k; /* strict '>' keeps the first maximum */
    return best;
}

/* ---------------------------------------------------------------------------
 * Sub-pixel 3-point fit along one axis (S8c "PIV step by step", step 3).
 * cm, c0, cp are the scores at d*-1, d*, d*+1.  Returns delta; sets *parabola
 * when the Gaussian fit was not applicable (some score <= 0).
 * ------------------------------------------------------------------------- */
double oracle_subpixel3(double cm, double c0, double cp, int *parabola)
{
    double num, den;
    if (cm > 0.0 && c0 > 0.0 && cp > 0.0) {
        /* Gaussian: delta = (ln c- - ln c+) / (2 (ln c- - 2 ln c0 + ln c+)) */
        const double lm = log(cm), l0 = log(c0), lp = log(cp);
        num = lm - lp;
        den = 2.0 * (lm - 2.0 * l0 + lp);
        *parabola = 0;
    } else {
        /* parabolic fallback: delta = (c- - c+) / (2 (c- - 2 c0 + c+)) */
        num = cm - cp;
        den = 2.0 * (cm - 2.0 * c0 + cp);
        *parabola = 1;
    }
    if (den >= 0.0) return 0.0; /* not a maximum (or flat): no fit */
    return num / den;
}

/* ---------------------------------------------------------------------------
 * Sub-pixel 3-point fit of a MINIMUM along one axis (SSD, the paper's PIV score: Fig 5.10
 * caption P:167-168 "offset sum of squared differences"; S8c reading 6): the parabola
 * through (-1, cm), (0, c0), (+1, cp) has its vertex at delta = (c- - c+) / (2 (c- - 2 c0 + c+));
 * it is a minimum only when that denominator is > 0, otherwise no fit (delta = 0).
 * ------------------------------------------------------------------------- */
double oracle_subpixel3_min(double cm, double c0, double cp)
{
    const double den = 2.0 * (cm - 2.0 * c0 + cp);
    if (den <= 0.0) return 0.0; /* not a minimum (or flat): no fit */
    return (cm - cp) / den;
}

typedef struct {
    int32_t iy, ix;  /* integer displacement of the peak (dy*, dx*)         */
    double dy, dx;   /* sub-pixel displacement dy* + delta_y, dx* + delta_x */
    double score;    /* NCC at the integer peak                            */
    uint32_t flags;  /* OF_* bits                                          */
} oracle_piv_vector;

/* One interrogation window: template A[y:y+h, x:x+w]; candidates B[y+dy.., x+dx..].
 * scratch holds (2my+1)*(2mx+1) doubles. */
static void piv_one_window(const float *A, const float *B, int64_t pitch,
                           int h, int w, int my, int mx, int y, int x,
                           double *scratch, oracle_piv_vector *out)
{
    const int OY = 2 * my + 1, OX = 2 * mx + 1;
    const float *tmpl = A + (int64_t)y * pitch + x;
    for (int dy = -my; dy <= my; ++dy)
        for (int dx = -mx; dx <= mx; ++dx)
            scratch[(dy + my) * OX + (dx + mx)] =
                corr2_window(B, pitch, y + dy, x + dx, tmpl, pitch, h, w);
    const int64_t k = oracle_argmax(scratch, (int64_t)OY * OX); /* tie -> row-major first */
    const int iy = (int)(k / OX) - my, ix = (int)(k % OX) - mx;
    uint32_t flags = 0;
    if (oracle_template_is_flat(tmpl, pitch, h, w)) flags |= OF_FLAT_TEMPLATE | OF_INVALID;
    double ddy = 0.0, ddx = 0.0;
    int par;
    if (iy == -my || iy == my) {
        flags |= OF_EDGE_Y;
    } else {
        ddy = oracle_subpixel3(scratch[(iy + my - 1) * OX + (ix + mx)],
                               scratch[(iy + my) * OX + (ix + mx)],
                               scratch[(iy + my + 1) * OX + (ix + mx)], &par);
        if (par) flags |= OF_PARABOLA_Y;
    }
    if (ix == -mx || ix == mx) {
        flags |= OF_EDGE_X;
    } else {
        ddx = oracle_subpixel3(scratch[(iy + my) * OX + (ix + mx - 1)],
                               scratch[(iy + my) * OX + (ix + mx)],
                               scratch[(iy + my) * OX + (ix + mx + 1)], &par);
        if (par) flags |= OF_PARABOLA_X;
    }
    out->iy = iy;
    out->ix = ix;
    out->dy = iy + ddy;
    out->dx = ix + ddx;
    out->score = scratch[k];
    out->flags = flags;
}

/* PIV with a distance score -- SSD (the paper's metric, Fig 5.10) or SAD: argmin over the search range
 * (tie -> smallest row-major index), 3-point parabolic sub-pixel fit of the minimum per axis
 * (delta = (c- - c+) / (2 (c- - 2 c0 + c+)), 0 if that denominator <= 0), no fit on the border. */
typedef double (*window_score_fn)(const float *, int64_t, int, int, const float *, int64_t, int, int);

static void piv_one_window_min(window_score_fn score, const float *A, const float *B, int64_t pitch,
                               int h, int w, int my, int mx, int y, int x,
                               double *scratch, oracle_piv_vector *out)
{
    const int OY = 2 * my + 1, OX = 2 * mx + 1;
    const float *tmpl = A + (int64_t)y * pitch + x;
    for (int dy = -my; dy <= my; ++dy)
        for (int dx = -mx; dx <= mx; ++dx)
            scratch[(dy + my) * OX + (dx + mx)] =
                score(B, pitch, y + dy, x + dx, tmpl, pitch, h, w);
    const int64_t k = oracle_argmin(scratch, (int64_t)OY * OX);
    const int iy = (int)(k / OX) - my, ix = (int)(k % OX) - mx;
    uint32_t flags = 0;
    double ddy = 0.0, ddx = 0.0;
    if (iy == -my || iy == my) {
        flags |= OF_EDGE_Y;
    } else {
        ddy = oracle_subpixel3_min(scratch[(iy + my - 1) * OX + (ix + mx)], scratch[(iy + my) * OX + (ix + mx)],
                                   scratch[(iy + my + 1) * OX + (ix + mx)]);
    }
    if (ix == -mx || ix == mx) {
        flags |= OF_EDGE_X;
    } else {
        ddx = oracle_subpixel3_min(scratch[(iy + my) * OX + (ix + mx - 1)], scratch[(iy + my) * OX + (ix + mx)],
                                   scratch[(iy + my) * OX + (ix + mx + 1)]);
    }
    out->iy = iy;
    out->ix = ix;
    out->dy = iy + ddy;
    out->dx = ix + ddx;
    out->score = scratch[k];
    out->flags = flags;
}

/* Window grid (S8 notation): K = floor((S - w - 2m)/s) + 1 per axis, window (ky,kx)
 * has its A-origin at (my + ky*sy, mx + kx*sx).  Interior windows only (S8c #9). */
int oracle_piv_grid(int H, int W, int h, int w, int my, int mx, int sy, int sx,
                    int *Ky, int *Kx)
{
    if (h <= 0 || w <= 0 || my < 0 || mx < 0 || sy <= 0 || sx <= 0) return -1;
    if (H - h - 2 * my < 0 || W - w - 2 * mx < 0) return -1;
    *Ky = (H - h - 2 * my) / sy + 1;
    *Kx = (W - w - 2 * mx) / sx + 1;
    return 0;
}

/* All windows of one frame pair: out[ky*Kx + kx]. scratch: nthreads*(2my+1)*(2mx+1)
 * doubles are allocated per window on the stack-free heap by the caller via
 * 'scratch' of size Ky*Kx*(2my+1)*(2mx+1) -- simplest possible ownership. */
int oracle_piv_pair(const float *A, const float *B, int H, int W, int64_t pitch,
                    int h, int w, int my, int mx, int sy, int sx,
                    double *scratch, oracle_piv_vector *out)
{
    int Ky, Kx;
    if (oracle_piv_grid(H, W, h, w, my, mx, sy, sx, &Ky, &Kx)) return -1;
    const int64_t per = (int64_t)(2 * my + 1) * (2 * mx + 1);
#pragma omp parallel for schedule(dynamic, 1)
    for (int k = 0; k < Ky * Kx; ++k) {
        const int ky = k / Kx, kx = k % Kx;
        piv_one_window(A, B, pitch, h, w, my, mx, my + ky * sy, mx + kx * sx,
                       scratch + (int64_t)k * per, &out[k]);
    }
    return 0;
}

/* Selected windows only (sampled parity at full size): windows (kys[i], kxs[i]).
 * scratch: count*(2my+1)*(2mx+1) doubles. */
int oracle_piv_windows(const float *A, const float *B, int H, int W, int64_t pitch,
                       int h, int w, int my, int mx, int sy, int sx,
                       const int *kys, const int *kxs, int count,
                       double *scratch, oracle_piv_vector *out)
{
    int Ky, Kx;
    if (oracle_piv_grid(H, W, h, w, my, mx, sy, sx, &Ky, &Kx)) return -1;
    for (int i = 0; i < count; ++i)
        if (kys[i] < 0 || kys[i] >= Ky || kxs[i] < 0 || kxs[i] >= Kx) return -1;
    const int64_t per = (int64_t)(2 * my + 1) * (2 * mx + 1);
#pragma omp parallel for schedule(dynamic, 1)
    for (int i = 0; i < count; ++i)
        piv_one_window(A, B, pitch, h, w, my, mx, my + kys[i] * sy, mx + kxs[i] * sx,
                       scratch + (int64_t)i * per, &out[i]);
    return 0;
}

/* Full PIV score surface of one window (for element-wise score parity tests). */
int oracle_piv_window_scores(const float *A, const float *B, int H, int W, int64_t pitch,
                             int h, int w, int my, int mx, int sy, int sx,
                             int ky, int kx, double *scores)
{
    int Ky, Kx;
    if (oracle_piv_grid(H, W, h, w, my, mx, sy, sx, &Ky, &Kx)) return -1;
    if (ky < 0 || ky >= Ky || kx < 0 || kx >= Kx) return -1;
    const int y = my + ky * sy, x = mx + kx * sx, OX = 2 * mx + 1;
    const float *tmpl = A + (int64_t)y * pitch + x;
    for (int dy = -my; dy <= my; ++dy)
        for (int dx = -mx; dx <= mx; ++dx)
            scores[(dy + my) * OX + (dx + mx)] =
                corr2_window(B, pitch, y + dy, x + dx, tmpl, pitch, h, w);
    return 0;
}

int oracle_piv_windows_ssd(const float *A, const float *B, int H, int W, int64_t pitch,
                           int h, int w, int my, int mx, int sy, int sx,
                           const int *kys, const int *kxs, int count,
                           double *scratch, oracle_piv_vector *out)
{
    int Ky, Kx;
    if (oracle_piv_grid(H, W, h, w, my, mx, sy, sx, &Ky, &Kx)) return -1;
    for (int i = 0; i < count; ++i)
        if (kys[i] < 0 || kys[i] >= Ky || kxs[i] < 0 || kxs[i] >= Kx) return -1;
    const int64_t per = (int64_t)(2 * my + 1) * (2 * mx + 1);
#pragma omp parallel for schedule(dynamic, 1)
    for (int i = 0; i < count; ++i)
        piv_one_window_min(ssd_window, A, B, pitch, h, w, my, mx, my + kys[i] * sy, mx + kxs[i] * sx,
                           scratch + (int64_t)i * per, &out[i]);
    return 0;
}

int oracle_piv_windows_sad(const float *A, const float *B, int H, int W, int64_t pitch,
                           int h, int w, int my, int mx, int sy, int sx,
                           const int *kys, const int *kxs, int count,
                           double *scratch, oracle_piv_vector *out)
{
    int Ky, Kx;
    if (oracle_piv_grid(H, W, h, w, my, mx, sy, sx, &Ky, &Kx)) return -1;
    for (int i = 0; i < count; ++i)
        if (kys[i] < 0 || kys[i] >= Ky || kxs[i] < 0 || kxs[i] >= Kx) return -1;
    const int64_t per = (int64_t)(2 * my + 1) * (2 * mx + 1);
#pragma omp parallel for schedule(dynamic, 1)
    for (int i = 0; i < count; ++i)
        piv_one_window_min(sad_window, A, B, pitch, h, w, my, mx, my + kys[i] * sy, mx + kxs[i] * sx,
                           scratch + (int64_t)i * per, &out[i]);
    return 0;
}

/* Set the OpenMP thread count of later calls (bench.py's 1-thread oracle rate). */
void oracle_set_num_threads(int n)
{
#ifdef _OPENMP
    extern void omp_set_num_threads(int);
    if (n > 0) omp_set_num_threads(n);
#else
    (void)n;
#endif
}

int oracle_num_threads(void)
{
#ifdef _OPENMP
    extern int omp_get_max_threads(void);
    return omp_get_max_threads();
#else
    return 1;
#endif
}

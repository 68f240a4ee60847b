/*
 * czc_oracle.c — CPU ORACLE (test infrastructure only; see czc_oracle.h for the contract).
 *
 * Plain definitions, no blocking, fusion or running sums.  Per-element arithmetic in double,
 * every sum in long double, moments two-pass centred.  Build:  gcc -O2 -fopenmp
 * -ffp-contract=off (no FMA contraction, IEEE round-to-nearest; reading R21).  OpenMP only
 * splits independent rows / window planes; their long-double partials are combined in index
 * order, so the result does not depend on the thread count beyond long-double rounding.
 */
#include "czc_oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

typedef long double ld;

int czco_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

/* Right-align a shape into (nz, ny, nx); returns 0 if invalid. */
static int shape3(int ndim, const int64_t* dims, int64_t n3[3]) {
  if (ndim < 1 || ndim > 3 || !dims) return 0;
  n3[0] = n3[1] = n3[2] = 1;
  for (int i = 0; i < ndim; i++) {
    if (dims[i] < 1) return 0;
    n3[3 - ndim + i] = dims[i];
  }
  return 1;
}

/* An input field: float32 (the paper's precision, L330) or float64 (NEXT row f3).  Every sample
 * is read as a double (float -> double is exact), so one definition serves both element types. */
typedef struct {
  const void* p;
  int f64;
} fld_t;
static inline fld_t fld32(const float* p) { fld_t f = {p, 0}; return f; }
static inline fld_t fld64(const double* p) { fld_t f = {p, 1}; return f; }
static inline double V(fld_t f, int64_t i) {
  return f.f64 ? ((const double*)f.p)[i] : (double)((const float*)f.p)[i];
}

/* e = recon - orig (reading R1), computed as (double)y - (double)x. */
static inline double err_of(fld_t x, fld_t y, int64_t i) {
  return V(y, i) - V(x, i);
}

/* ======================================================================================
 * Pattern 1 — global reductions.  Table I Category I (L107): min/max/avg error, pwr error,
 * MSE, RMSE, NRMSE, SNR, PSNR; plus north_star's range, max relative error and Pearson.
 * Definitions: SURVEY.md §8(c) C-P1 and readings R1-R6.
 * ====================================================================================== */
static int p1_impl(fld_t x, fld_t y, uint64_t n, czco_p1_t* r) {
  if (!x.p || !y.p || !r || n == 0) return 1;
  memset(r, 0, sizeof(*r));
  /* pass 1: extrema, plain sums */
  double xmin = V(x, 0), xmax = xmin;
  double emin = err_of(x, y, 0), emax = emin, emaxabs = fabs(emin);
  double pmin = INFINITY, pmax = -INFINITY;
  uint64_t npwr = 0;
  ld sx = 0, sy = 0, se = 0, sae = 0, spwr = 0;
  for (uint64_t i = 0; i < n; i++) {
    const double xi = V(x, (int64_t)i);
    double e = err_of(x, y, (int64_t)i);
    if (xi < xmin) xmin = xi;
    if (xi > xmax) xmax = xi;
    if (e < emin) emin = e;
    if (e > emax) emax = e;
    if (fabs(e) > emaxabs) emaxabs = fabs(e);
    sx += (ld)xi;
    sy += (ld)V(y, (int64_t)i);
    se += (ld)e;
    sae += (ld)fabs(e);
    if (xi != 0.0) {                       /* point-wise relative error, x = 0 excluded (R3) */
      double q = fabs(e) / fabs(xi);
      if (q < pmin) pmin = q;
      if (q > pmax) pmax = q;
      spwr += (ld)q;
      npwr++;
    }
  }
  const ld N = (ld)n;
  const ld mx = sx / N, my = sy / N, me = se / N;
  /* pass 2: centred second moments */
  ld sxx = 0, syy = 0, sxy = 0, svar = 0, se2 = 0;
  for (uint64_t i = 0; i < n; i++) {
    ld dx = (ld)V(x, (int64_t)i) - mx, dy = (ld)V(y, (int64_t)i) - my;
    ld e = (ld)err_of(x, y, (int64_t)i);
    sxx += dx * dx;
    syy += dy * dy;
    sxy += dx * dy;
    svar += (e - me) * (e - me);
    se2 += e * e;
  }
  r->n = n;
  r->x_min = xmin;
  r->x_max = xmax;
  r->value_range = xmax - xmin;                      /* R4: range of the original */
  r->err_min = emin;
  r->err_max = emax;
  r->err_maxabs = emaxabs;
  r->err_mean = (double)me;
  r->err_absmean = (double)(sae / N);
  const ld mse = se2 / N;
  r->mse = (double)mse;
  r->rmse = (double)sqrtl(mse);
  const double R = r->value_range;
  r->nrmse = (R > 0) ? (double)(sqrtl(mse) / (ld)R) : (mse > 0 ? INFINITY : NAN);
  if (mse == 0) r->psnr = INFINITY;                  /* zero error: PSNR = +inf (north_star) */
  else if (R == 0) r->psnr = -INFINITY;
  else r->psnr = (double)(20.0L * log10l((ld)R) - 10.0L * log10l(mse));
  /* R5: SNR = 10 log10( sum (x - mean x)^2 / sum e^2 ) */
  if (se2 == 0) r->snr = (sxx > 0) ? INFINITY : NAN;
  else r->snr = (double)(10.0L * log10l(sxx / se2));
  r->max_rel_err = (R > 0) ? emaxabs / R : (emaxabs > 0 ? INFINITY : NAN);
  r->n_pwr = npwr;
  r->pwr_min = npwr ? pmin : NAN;
  r->pwr_max = npwr ? pmax : NAN;
  r->pwr_mean = npwr ? (double)(spwr / (ld)npwr) : NAN;
  r->pearson = (sxx > 0 && syy > 0) ? (double)(sxy / sqrtl(sxx * syy)) : NAN;
  r->err_var = (double)(svar / N);                   /* R6: population variance */
  return 0;
}
int czco_p1(const float* x, const float* y, uint64_t n, czco_p1_t* r) { return p1_impl(fld32(x), fld32(y), n, r); }
int czco_p1_f64(const double* x, const double* y, uint64_t n, czco_p1_t* r) {
  return p1_impl(fld64(x), fld64(y), n, r);
}

/* ======================================================================================
 * Pattern 2 — stencil metrics.  Eq. (1): Der = sum_a |f(p+e_a) - f(p-e_a)|;  "the
 * Divergence and Laplacian metrics are the sums of first- and second-order derivatives" (L129);
 * Alg. 2: central differences /2 and their L2 norm (Grad).  Readings R7, R9, R11:
 * interior points only (1-point border on every active axis), compact second difference.
 * ====================================================================================== */
static void deriv_point(fld_t f, const int64_t n3[3], const int act[3], int64_t z, int64_t yy,
                        int64_t xx, double F[CZCO_NF]) {
  const int64_t st[3] = {n3[1] * n3[2], n3[2], 1};
  const int64_t c = z * st[0] + yy * st[1] + xx;
  const double f0 = V(f, c);
  double der1 = 0, der2 = 0, g2 = 0, div = 0, lap = 0;
  for (int a = 0; a < 3; a++) {
    if (!act[a]) continue;
    const double fp = V(f, c + st[a]), fm = V(f, c - st[a]);
    const double delta = fp - fm;               /* first difference f(p+1) - f(p-1)      */
    const double D = delta / 2.0;               /* central derivative (Alg. 2)  */
    const double lap_a = fp - 2.0 * f0 + fm;    /* second difference f(p+1)-2f(p)+f(p-1)  */
    der1 += fabs(delta);
    der2 += fabs(lap_a);
    g2 += D * D;
    div += D;
    lap += lap_a;
  }
  F[CZCO_DER1] = der1;
  F[CZCO_DER2] = der2;
  F[CZCO_GRAD] = sqrt(g2);
  F[CZCO_DIV] = div;
  F[CZCO_LAP] = lap;
}

static int deriv_impl(fld_t x, fld_t y, int ndim, const int64_t* dims, czco_deriv_t* r) {
  int64_t n3[3];
  if (!x.p || !y.p || !r || !shape3(ndim, dims, n3)) return 1;
  memset(r, 0, sizeof(*r));
  int act[3], any = 0;
  int64_t lo[3], hi[3];
  for (int a = 0; a < 3; a++) {
    act[a] = n3[a] > 1;
    any |= act[a];
    lo[a] = act[a] ? 1 : 0;
    hi[a] = act[a] ? n3[a] - 1 : 1;            /* exclusive */
  }
  int64_t nI = 1;
  for (int a = 0; a < 3; a++) nI *= (hi[a] > lo[a]) ? (hi[a] - lo[a]) : 0;
  if (!any) nI = 0;
  r->n_interior = (uint64_t)nI;
  const int64_t nrows = (hi[0] > lo[0] ? hi[0] - lo[0] : 0) * (hi[1] > lo[1] ? hi[1] - lo[1] : 0);
  /* per-row partials (one row = fixed z, y), combined in row order */
  ld* psa = calloc((size_t)(nrows > 0 ? nrows : 1) * CZCO_NF * 2, sizeof(ld));
  double* pext = malloc((size_t)(nrows > 0 ? nrows : 1) * CZCO_NF * 3 * sizeof(double));
  if (!psa || !pext) { free(psa); free(pext); return 2; }
  const int64_t ny_i = hi[1] - lo[1];
#pragma omp parallel for schedule(dynamic, 4)
  for (int64_t row = 0; row < nrows; row++) {
    const int64_t z = lo[0] + row / ny_i, yy = lo[1] + row % ny_i;
    ld* sa = psa + row * CZCO_NF * 2;
    double* ex = pext + row * CZCO_NF * 3;
    for (int k = 0; k < CZCO_NF; k++) { ex[3 * k] = 0; ex[3 * k + 1] = INFINITY; ex[3 * k + 2] = -INFINITY; }
    for (int64_t xx = lo[2]; xx < hi[2]; xx++) {
      double Fx[CZCO_NF], Fy[CZCO_NF];
      deriv_point(x, n3, act, z, yy, xx, Fx);
      deriv_point(y, n3, act, z, yy, xx, Fy);
      for (int k = 0; k < CZCO_NF; k++) {
        const double d = Fy[k] - Fx[k];        /* error of the derived field */
        if (fabs(d) > ex[3 * k]) ex[3 * k] = fabs(d);
        if (Fx[k] < ex[3 * k + 1]) ex[3 * k + 1] = Fx[k];
        if (Fx[k] > ex[3 * k + 2]) ex[3 * k + 2] = Fx[k];
        sa[2 * k] += (ld)fabs(d);
        sa[2 * k + 1] += (ld)d * (ld)d;
      }
    }
  }
  for (int k = 0; k < CZCO_NF; k++) {
    ld s1 = 0, s2 = 0;
    double mx = 0, fmn = INFINITY, fmx = -INFINITY;
    for (int64_t row = 0; row < nrows; row++) {
      s1 += psa[row * CZCO_NF * 2 + 2 * k];
      s2 += psa[row * CZCO_NF * 2 + 2 * k + 1];
      const double* ex = pext + row * CZCO_NF * 3 + 3 * k;
      if (ex[0] > mx) mx = ex[0];
      if (ex[1] < fmn) fmn = ex[1];
      if (ex[2] > fmx) fmx = ex[2];
    }
    czco_deriv_field_t* o = &r->f[k];
    if (nI == 0) {
      o->maxabs = o->mae = o->mse = o->rmse = o->f_min = o->f_max = o->psnr = NAN;
      continue;
    }
    const ld mse = s2 / (ld)nI;
    o->maxabs = mx;
    o->mae = (double)(s1 / (ld)nI);
    o->mse = (double)mse;
    o->rmse = (double)sqrtl(mse);
    o->f_min = fmn;
    o->f_max = fmx;
    const double rng = fmx - fmn;
    if (mse == 0) o->psnr = INFINITY;
    else if (rng == 0) o->psnr = -INFINITY;
    else o->psnr = (double)(20.0L * log10l((ld)rng) - 10.0L * log10l(mse));
  }
  free(psa);
  free(pext);
  return 0;
}
int czco_deriv(const float* x, const float* y, int ndim, const int64_t* dims, czco_deriv_t* r) {
  return deriv_impl(fld32(x), fld32(y), ndim, dims, r);
}
int czco_deriv_f64(const double* x, const double* y, int ndim, const int64_t* dims, czco_deriv_t* r) {
  return deriv_impl(fld64(x), fld64(y), ndim, dims, r);
}

/* ======================================================================================
 * Error autocorrelation, Eq. (2):
 *   AC(tau) = [ sum_{p in R_tau} (e_p - mu) * (1/D) sum_a (e_{p+tau e_a} - mu) ] / ne / sigma^2
 * R_tau = { p : p_a <= n_a - 1 - tau on every active axis },  ne = prod_a (n_a - tau).
 * mu, sigma^2: mean and (population) variance of e over all N elements (R13).  1/3 -> 1/D (R12).
 * ====================================================================================== */
static int autocorr_impl(fld_t x, fld_t y, int ndim, const int64_t* dims, int max_lag,
                         double* ac, uint64_t* count) {
  int64_t n3[3];
  if (!x.p || !y.p || !ac || !count || max_lag < 0 || !shape3(ndim, dims, n3)) return 1;
  const int64_t N = n3[0] * n3[1] * n3[2];
  const int64_t st[3] = {n3[1] * n3[2], n3[2], 1};
  int act[3], D = 0;
  int64_t nmin = INT64_MAX;
  for (int a = 0; a < 3; a++) {
    act[a] = n3[a] > 1;
    D += act[a];
    if (act[a] && n3[a] < nmin) nmin = n3[a];
  }
  ld se = 0;
  for (int64_t i = 0; i < N; i++) se += (ld)err_of(x, y, i);
  const ld mu = se / (ld)N;
  ld sv = 0;
  for (int64_t i = 0; i < N; i++) {
    const ld d = (ld)err_of(x, y, i) - mu;
    sv += d * d;
  }
  const ld var = sv / (ld)N;
  ac[0] = 1.0;
  count[0] = (uint64_t)N;
  for (int tau = 1; tau <= max_lag; tau++) {
    if (D == 0 || tau >= nmin) { ac[tau] = NAN; count[tau] = 0; continue; }
    int64_t hi[3];
    int64_t ne = 1;
    for (int a = 0; a < 3; a++) {
      hi[a] = act[a] ? n3[a] - tau : 1;         /* p_a in [0, hi_a) */
      ne *= hi[a];
    }
    count[tau] = (uint64_t)ne;
    const int64_t nrows = hi[0] * hi[1];
    ld* part = calloc((size_t)nrows, sizeof(ld));
    if (!part) return 2;
#pragma omp parallel for schedule(dynamic, 8)
    for (int64_t row = 0; row < nrows; row++) {
      const int64_t z = row / hi[1], yy = row % hi[1];
      ld s = 0;
      for (int64_t xx = 0; xx < hi[2]; xx++) {
        const int64_t p = z * st[0] + yy * st[1] + xx;
        const ld ep = (ld)err_of(x, y, p) - mu;
        ld nb = 0;
        for (int a = 0; a < 3; a++)
          if (act[a]) nb += (ld)err_of(x, y, p + (int64_t)tau * st[a]) - mu;
        s += ep * (nb / (ld)D);
      }
      part[row] = s;
    }
    ld tot = 0;
    for (int64_t row = 0; row < nrows; row++) tot += part[row];
    free(part);
    ac[tau] = (var > 0) ? (double)(tot / (ld)ne / var) : NAN;
  }
  return 0;
}
int czco_autocorr(const float* x, const float* y, int ndim, const int64_t* dims, int max_lag,
                  double* ac, uint64_t* count) {
  return autocorr_impl(fld32(x), fld32(y), ndim, dims, max_lag, ac, count);
}
int czco_autocorr_f64(const double* x, const double* y, int ndim, const int64_t* dims, int max_lag,
                      double* ac, uint64_t* count) {
  return autocorr_impl(fld64(x), fld64(y), ndim, dims, max_lag, ac, count);
}

/* ======================================================================================
 * SSIM, L139-L146: a w^D window slides with a fixed step over both fields; per window the
 * min, max, sum and power sums give the local SSIM (Wang et al. [25], K1=0.01, K2=0.03,
 * C3=C2/2 — R14); the final SSIM is the mean of all local SSIMs (L146, R16).  Valid windows
 * only (o_a + w_a <= n_a, R17).  Dynamic range L = max - min of the ORIGINAL window (R15;
 * range_mode 1: the caller's global range), L := 1 when L == 0.
 * ====================================================================================== */
static double ssim_window3(fld_t x, fld_t y, const int64_t n3[3], const int64_t o[3],
                           const int64_t w[3], int range_mode, double global_range) {
  const int64_t st[3] = {n3[1] * n3[2], n3[2], 1};
  const ld M = (ld)(w[0] * w[1] * w[2]);
  ld sx = 0, sy = 0;
  double xmin = V(x, o[0] * st[0] + o[1] * st[1] + o[2]), xmax = xmin;
  for (int64_t k = 0; k < w[0]; k++)
    for (int64_t j = 0; j < w[1]; j++)
      for (int64_t i = 0; i < w[2]; i++) {
        const int64_t p = (o[0] + k) * st[0] + (o[1] + j) * st[1] + o[2] + i;
        const double xp = V(x, p);
        sx += (ld)xp;
        sy += (ld)V(y, p);
        if (xp < xmin) xmin = xp;
        if (xp > xmax) xmax = xp;
      }
  const ld mx = sx / M, my = sy / M;
  ld vx = 0, vy = 0, cxy = 0;
  for (int64_t k = 0; k < w[0]; k++)
    for (int64_t j = 0; j < w[1]; j++)
      for (int64_t i = 0; i < w[2]; i++) {
        const int64_t p = (o[0] + k) * st[0] + (o[1] + j) * st[1] + o[2] + i;
        const ld dx = (ld)V(x, p) - mx, dy = (ld)V(y, p) - my;
        vx += dx * dx;
        vy += dy * dy;
        cxy += dx * dy;
      }
  vx /= M;
  vy /= M;
  cxy /= M;
  ld L = range_mode ? (ld)global_range : (ld)xmax - (ld)xmin;
  if (L == 0) L = 1;
  const ld C1 = (0.01L * L) * (0.01L * L), C2 = (0.03L * L) * (0.03L * L);
  const ld num = (2 * mx * my + C1) * (2 * cxy + C2);
  const ld den = (mx * mx + my * my + C1) * (vx + vy + C2);
  return (double)(num / den);
}

static int window3(int ndim, const int64_t* v, int64_t out[3], int64_t fill) {
  out[0] = out[1] = out[2] = fill;
  for (int i = 0; i < ndim; i++) out[3 - ndim + i] = v[i];
  return 1;
}

static double ssim_window_impl(fld_t x, fld_t y, int ndim, const int64_t* dims,
                               const int64_t* origin, const int64_t* window, int range_mode,
                               double global_range) {
  int64_t n3[3], o[3], w[3];
  if (!x.p || !y.p || !shape3(ndim, dims, n3)) return NAN;
  window3(ndim, origin, o, 0);
  window3(ndim, window, w, 1);
  for (int a = 0; a < 3; a++) {
    if (n3[a] == 1) w[a] = 1;                   /* inactive axis: extent 1 */
    if (w[a] < 1 || o[a] < 0 || o[a] + w[a] > n3[a]) return NAN;
  }
  return ssim_window3(x, y, n3, o, w, range_mode, global_range);
}
double czco_ssim_window(const float* x, const float* y, int ndim, const int64_t* dims,
                        const int64_t* origin, const int64_t* window, int range_mode,
                        double global_range) {
  return ssim_window_impl(fld32(x), fld32(y), ndim, dims, origin, window, range_mode, global_range);
}
double czco_ssim_window_f64(const double* x, const double* y, int ndim, const int64_t* dims,
                            const int64_t* origin, const int64_t* window, int range_mode,
                            double global_range) {
  return ssim_window_impl(fld64(x), fld64(y), ndim, dims, origin, window, range_mode, global_range);
}

static int ssim_impl(fld_t x, fld_t y, int ndim, const int64_t* dims, const int64_t* window,
                     const int64_t* step, int range_mode, double* ssim, uint64_t* n_windows) {
  int64_t n3[3], w[3], s[3], nw[3];
  if (!x.p || !y.p || !ssim || !n_windows || !shape3(ndim, dims, n3)) return 1;
  window3(ndim, window, w, 1);
  window3(ndim, step, s, 1);
  double grange = 0;
  if (range_mode) {
    const int64_t N = n3[0] * n3[1] * n3[2];
    double mn = V(x, 0), mxv = mn;
    for (int64_t i = 0; i < N; i++) {
      const double v = V(x, i);
      if (v < mn) mn = v;
      if (v > mxv) mxv = v;
    }
    grange = mxv - mn;
  }
  for (int a = 0; a < 3; a++) {
    if (n3[a] == 1) { w[a] = 1; s[a] = 1; }
    if (w[a] < 1 || s[a] < 1) return 1;
    nw[a] = (w[a] <= n3[a]) ? (n3[a] - w[a]) / s[a] + 1 : 0;
  }
  const int64_t total = nw[0] * nw[1] * nw[2];
  *n_windows = (uint64_t)total;
  if (total == 0) { *ssim = NAN; return 3; }   /* no valid window: shape error (R16) */
  const int64_t nrows = nw[0] * nw[1];
  ld* part = calloc((size_t)nrows, sizeof(ld));
  if (!part) return 2;
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t row = 0; row < nrows; row++) {
    int64_t o[3] = {(row / nw[1]) * s[0], (row % nw[1]) * s[1], 0};
    ld acc = 0;
    for (int64_t i = 0; i < nw[2]; i++) {
      o[2] = i * s[2];
      acc += (ld)ssim_window3(x, y, n3, o, w, range_mode, grange);
    }
    part[row] = acc;
  }
  ld tot = 0;
  for (int64_t row = 0; row < nrows; row++) tot += part[row];
  free(part);
  *ssim = (double)(tot / (ld)total);
  return 0;
}
int czco_ssim(const float* x, const float* y, int ndim, const int64_t* dims, const int64_t* window,
              const int64_t* step, int range_mode, double* ssim, uint64_t* n_windows) {
  return ssim_impl(fld32(x), fld32(y), ndim, dims, window, step, range_mode, ssim, n_windows);
}
int czco_ssim_f64(const double* x, const double* y, int ndim, const int64_t* dims, const int64_t* window,
                  const int64_t* step, int range_mode, double* ssim, uint64_t* n_windows) {
  return ssim_impl(fld64(x), fld64(y), ndim, dims, window, step, range_mode, ssim, n_windows);
}

/* ======================================================================================
 * Error PDF / pwr-error PDF (Table I Category I, L107).  The paper names the two metrics but
 * defines no binning; reading R24: equal-width bins over the value range of the data.
 * Pass 1 finds the ranges (the same extrema as czco_p1), pass 2 bins every value.
 * ====================================================================================== */
static int pdf_bin(double v, double lo, double w, int nbins) {
  if (!(w > 0) || isinf(w)) return 0;
  const double q = (v - lo) / w;              /* IEEE quotient, no contraction (R21) */
  int b = (int)floor(q);
  if (b >= nbins) b = nbins - 1;
  if (b < 0) b = 0;
  return b;
}

static int pdf_impl(fld_t x, fld_t y, uint64_t n, int nbins, double* err_lo, double* err_w,
                    uint64_t* err_counts, double* pwr_lo, double* pwr_w, uint64_t* pwr_counts, uint64_t* n_pwr) {
  if (!x.p || !y.p || n == 0 || nbins < 1 || !err_counts || !pwr_counts) return 1;
  double emin = INFINITY, emax = -INFINITY, pmin = INFINITY, pmax = -INFINITY;
  uint64_t np = 0;
  for (uint64_t i = 0; i < n; i++) {
    const double e = err_of(x, y, (int64_t)i);
    if (e < emin) emin = e;
    if (e > emax) emax = e;
    const double xi = V(x, (int64_t)i);
    if (xi != 0.0) {
      const double q = fabs(e) / fabs(xi);
      if (q < pmin) pmin = q;
      if (q > pmax) pmax = q;
      np++;
    }
  }
  const double ew = (emax - emin) / (double)nbins;
  const double pw = np ? (pmax - pmin) / (double)nbins : NAN;
  for (int b = 0; b < nbins; b++) err_counts[b] = pwr_counts[b] = 0;
  for (uint64_t i = 0; i < n; i++) {
    const double e = err_of(x, y, (int64_t)i);
    err_counts[pdf_bin(e, emin, ew, nbins)]++;
    const double xi = V(x, (int64_t)i);
    if (xi != 0.0) pwr_counts[pdf_bin(fabs(e) / fabs(xi), pmin, pw, nbins)]++;
  }
  *err_lo = emin;
  *err_w = ew;
  *pwr_lo = np ? pmin : NAN;
  *pwr_w = pw;
  *n_pwr = np;
  return 0;
}
int czco_pdf(const float* x, const float* y, uint64_t n, int nbins, double* err_lo, double* err_w,
             uint64_t* err_counts, double* pwr_lo, double* pwr_w, uint64_t* pwr_counts, uint64_t* n_pwr) {
  return pdf_impl(fld32(x), fld32(y), n, nbins, err_lo, err_w, err_counts, pwr_lo, pwr_w, pwr_counts, n_pwr);
}
int czco_pdf_f64(const double* x, const double* y, uint64_t n, int nbins, double* err_lo, double* err_w,
                 uint64_t* err_counts, double* pwr_lo, double* pwr_w, uint64_t* pwr_counts, uint64_t* n_pwr) {
  return pdf_impl(fld64(x), fld64(y), n, nbins, err_lo, err_w, err_counts, pwr_lo, pwr_w, pwr_counts, n_pwr);
}

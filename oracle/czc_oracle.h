/*
 * czc_oracle.h — CPU ORACLE for the cuZ-Checker assessment hot path.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
 * load this library.  It shares no code, header, table or helper with the CUDA path
 * (paper_conf_cluster_yudgtc21_b200/csrc); the two are compared field by field from Python.
 *
 * Every function is the plain definition of a metric from PAPER.md (Yu et al., CLUSTER'21),
 * written out with double per-element arithmetic and long-double (x87, 64-bit mantissa)
 * accumulation, two-pass centred moments, and brute-force per-window SSIM.  Where the paper is
 * silent or garbled the reading taken is SURVEY.md §8(c)'s register (R1..R23), listed again in
 * DESIGN.md §2.  Citations "Lnnn" are lines of PAPER.md.
 *
 * Shapes: ndim in 1..4 (4-D: NEXT row f3, L92), dims slowest-first, C order (x = last axis
 * contiguous).  Internally a shape is right-aligned into four axes with leading 1s; an axis with
 * n == 1 is "inactive" (it carries no stencil neighbour, no lag and a window extent of 1).
 * D = number of active axes.
 */
#ifndef CZC_ORACLE_H
#define CZC_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

/* Pattern 1, Table I Category I (L107, L111) + north_star list (range, max rel. err, Pearson). */
typedef struct {
  uint64_t n;
  double x_min, x_max, value_range;
  double err_min, err_max, err_maxabs, err_mean, err_absmean;
  double mse, rmse, nrmse, psnr, snr, max_rel_err;
  double pwr_min, pwr_max, pwr_mean;
  uint64_t n_pwr;
  double pearson, err_var;
} czco_p1_t;

/* Pattern 2 derived fields: Der1 (Eq. 1), Der2, Grad (Alg. 2), Div, Lap (L129). */
enum { CZCO_DER1 = 0, CZCO_DER2 = 1, CZCO_GRAD = 2, CZCO_DIV = 3, CZCO_LAP = 4, CZCO_NF = 5 };
typedef struct {
  double maxabs, mae, mse, rmse, f_min, f_max, psnr;
} czco_deriv_field_t;
typedef struct {
  uint64_t n_interior;
  czco_deriv_field_t f[CZCO_NF];
} czco_deriv_t;

/* returns 0 on success, nonzero on invalid arguments */
int czco_p1(const float* x, const float* y, uint64_t n, czco_p1_t* out);

int czco_deriv(const float* x, const float* y, int ndim, const int64_t* dims, czco_deriv_t* out);

/* Per-point errors dF = F(y) - F(x) of the five derived fields (Alg. 2 "Der"), out =
 * 5 x n_interior doubles, field-major, interior points in C order; returns 3 if no interior. */
int czco_deriv_points(const float* x, const float* y, int ndim, const int64_t* dims, double* out);
int czco_deriv_points_f64(const double* x, const double* y, int ndim, const int64_t* dims, double* out);

/* Eq. 2 (L133): ac[0..max_lag], count[0..max_lag] (= ne_tau).  mu, sigma^2 over all N elements. */
int czco_autocorr(const float* x, const float* y, int ndim, const int64_t* dims, int max_lag,
                  double* ac, uint64_t* count);

/* SSIM of one window (L139-L146), origin/extent given per input axis (slowest-first). */
double czco_ssim_window(const float* x, const float* y, int ndim, const int64_t* dims,
                        const int64_t* origin, const int64_t* window, int range_mode,
                        double global_range);

/* Global SSIM = mean of local SSIMs over all valid windows at multiples of step (L146). */
int czco_ssim(const float* x, const float* y, int ndim, const int64_t* dims, const int64_t* window,
              const int64_t* step, int range_mode, double* ssim, uint64_t* n_windows);

/* Separable SSIM (step 1, up to three active axes) for fields too large for the brute force;
 * the same definition as czco_ssim; *n_brute = windows recomputed by the brute force. */
int czco_ssim_separable(const float* x, const float* y, int ndim, const int64_t* dims, const int64_t* window,
                        int range_mode, double* ssim, uint64_t* n_windows, uint64_t* n_brute);
int czco_ssim_separable_f64(const double* x, const double* y, int ndim, const int64_t* dims, const int64_t* window,
                            int range_mode, double* ssim, uint64_t* n_windows, uint64_t* n_brute);

/* Local SSIM of every valid window, C order of the window-origin grid (out: n_windows doubles);
 * returns 3 when there is no valid window. */
int czco_ssim_windows(const float* x, const float* y, int ndim, const int64_t* dims, const int64_t* window,
                      const int64_t* step, int range_mode, double* out);
int czco_ssim_windows_f64(const double* x, const double* y, int ndim, const int64_t* dims, const int64_t* window,
                          const int64_t* step, int range_mode, double* out);

/* Error PDF and pwr-error PDF (Table I Category I, L107: "Error PDF", "Pwr error PDF"; the paper
 * gives no bin rule — reading R24): nbins equal-width bins over [min, max] of the
 * values (the error e = y - x over all n elements; |e|/|x| over x != 0), bin of v =
 * floor((v - lo) / w) with w = (max - min) / nbins, the top edge clamped into the last bin, w == 0
 * -> bin 0.  Outputs: lo, w and counts[nbins] of each; *n_pwr = number of x != 0 (if 0, the pwr
 * lo / w are NaN and its counts 0).  Returns 0 on success. */
int czco_pdf(const float* x, const float* y, uint64_t n, int nbins, double* err_lo, double* err_w,
             uint64_t* err_counts, double* pwr_lo, double* pwr_w, uint64_t* pwr_counts, uint64_t* n_pwr);

/* float64 inputs (NEXT row f3; the paper evaluates single precision only, L330): the same
 * definitions, every sample read as a double.  For float-representable data they return exactly
 * what the float32 entry points return. */
int czco_p1_f64(const double* x, const double* y, uint64_t n, czco_p1_t* out);
int czco_deriv_f64(const double* x, const double* y, int ndim, const int64_t* dims, czco_deriv_t* out);
int czco_autocorr_f64(const double* x, const double* y, int ndim, const int64_t* dims, int max_lag,
                      double* ac, uint64_t* count);
double czco_ssim_window_f64(const double* x, const double* y, int ndim, const int64_t* dims,
                            const int64_t* origin, const int64_t* window, int range_mode,
                            double global_range);
int czco_ssim_f64(const double* x, const double* y, int ndim, const int64_t* dims, const int64_t* window,
                  const int64_t* step, int range_mode, double* ssim, uint64_t* n_windows);
int czco_pdf_f64(const double* x, const double* y, uint64_t n, int nbins, double* err_lo, double* err_w,
                 uint64_t* err_counts, double* pwr_lo, double* pwr_w, uint64_t* pwr_counts, uint64_t* n_pwr);

/* Number of OpenMP threads the oracle uses (bench.py reports it as "cores"). */
int czco_threads(void);

#ifdef __cplusplus
}
#endif
#endif

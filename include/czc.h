/*
 * czc.h — C ABI of the B200-native cuZ-Checker assessment hot path.
 *
 * Paper: Yu, Di, Gok, Tao, Cappello, "cuZ-Checker: A GPU-Based Ultra-Fast Assessment System for
 * Lossy Compressions", IEEE CLUSTER 2021 (PAPER.md; "Lnnn" below = line nnn of PAPER.md).
 *
 * The paper's problem statement: data produced on the GPU is assessed "completely within the GPU
 * environment" without moving it to the CPU (abstract, L15; L33-L35).  A "GPU module coordinator
 * ... identifies the category of the user-requested metrics and then invokes the corresponding
 * optimized fused CUDA kernel" (L96); a GPU-compatible configuration parser supplies the settings
 * (L73, L75), e.g. the SSIM "window size and stride are defined by the user" (L139).
 *
 * Three pattern engines (Table I) sit behind one call:
 *   P1  global reduction  — min/max/range, errors, MSE/RMSE/NRMSE, SNR/PSNR, pwr error, Pearson
 *   P2  stencil-like      — derivative-family errors (Eq. 1; L129) and error
 *                           autocorrelation (Eq. 2)
 *   P3  sliding window    — 3-D (or 2-D) SSIM (L139-L146)
 * Metric definitions and every reading taken where the paper is silent: DESIGN.md §2.
 *
 * Conventions (all entry points):
 *   - Shapes: ndim 1..4, dims slowest-first, C order; the last axis is contiguous.  An axis of
 *     extent 1 is inactive (no stencil neighbour, no lag, window extent 1).  Fields with at most
 *     three active axes run on the streamed 3-D engines; four active axes (L92: "easily extended
 *     to ... 4D"; NEXT row f3) run generic grid-stride kernels (single GPU, no slab mode).
 *   - Every function returns czc_status; nothing aborts and no C++ exception crosses the ABI.
 *     On error, out->computed_mask = 0 and nothing else in *out is meaningful.
 *   - Undefined metrics are NaN (e.g. Pearson with zero variance, AC with sigma_e^2 = 0, pwr
 *     statistics with no non-zero original value); PSNR = +inf when MSE = 0.
 *   - Inputs are assumed finite; results for NaN/Inf inputs are unspecified.
 *   - A context is used by one host thread at a time.  Calls are synchronous: on return, *out is
 *     filled and the context's stream has no pending work of this call.
 */
#ifndef CZC_H
#define CZC_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define CZC_ABI_VERSION 5
#define CZC_MAX_DIMS 4           /* ndim 1..3 on the streamed engines; 4-D fields (NEXT row f3)    */
#define CZC_MAX_LAG 16           /* largest supported autocorrelation lag (paper uses <= 10, L345) */
#define CZC_PDF_MAX_BINS 256     /* largest number of error-PDF bins                              */

typedef enum czc_status {
  CZC_OK = 0,
  CZC_ERR_INVALID = 1,           /* NULL pointer, bad config value                              */
  CZC_ERR_SHAPE = 2,             /* ndim/dims invalid, SSIM window larger than the field, ...  */
  CZC_ERR_DTYPE = 3,             /* dtype not one of czc_dtype                                  */
  CZC_ERR_CUDA = 4,              /* a CUDA runtime call or kernel launch failed                 */
  CZC_ERR_NOMEM = 5,             /* device or host allocation failed                            */
  CZC_ERR_COMM = 6,              /* NCCL failure (multi-GPU slab mode)                          */
  CZC_ERR_UNSUPPORTED = 7        /* feature not built / requested combination not supported     */
} czc_status;

/* Element type of BOTH fields.  CZC_F32 is the paper's precision (L330: "all the data are
 * single-precision"); CZC_F64 is NEXT row f3 ("easily extended", L92): the same kernels with a
 * double element type (every accumulator is FP64 either way; e = y - x is rounded to double, as
 * in the oracle, reading R1), 16 bytes per element pair instead of 8. */
typedef enum czc_dtype { CZC_F32 = 0, CZC_F64 = 1 } czc_dtype;

/* metric_mask bits — one per pattern group (Table I categories, L107). */
enum {
  CZC_M_P1 = 1u << 0,            /* Category I: global reductions (L111)                        */
  CZC_M_DERIV = 1u << 1,         /* Category II: Der1/Der2/Grad/Div/Lap errors (L120-L129)      */
  CZC_M_AUTOCORR = 1u << 2,      /* Category II: error autocorrelation, Eq. 2 (L131-L135)        */
  CZC_M_SSIM = 1u << 3,          /* Category III: SSIM (L139-L146)                               */
  CZC_M_PDF = 1u << 4,           /* Category I: error PDF and pwr-error PDF (Table I): one */
                                 /* extra pass over the pair after P1 (bins span P1's extrema)  */
  CZC_M_ALL = 0xFu,              /* the four pattern groups of the north_star (bench.py's step) */
  CZC_M_FULL = 0x1Fu             /* every metric group, PDFs included                           */
};

/* Indices of czc_result.deriv[] */
enum { CZC_DER1 = 0, CZC_DER2 = 1, CZC_GRAD = 2, CZC_DIV = 3, CZC_LAP = 4, CZC_NDERIV = 5 };

typedef struct czc_config {
  int device;                    /* CUDA device ordinal the context binds to; -1 = current       */
  void* stream;                  /* cudaStream_t to run on; NULL = a BLOCKING stream owned by the */
                                 /* context (ordered after the caller's legacy-default-stream    */
                                 /* work, e.g. PyTorch's default stream, handle 0)               */
  int ssim_window[CZC_MAX_DIMS]; /* window extent per input axis (index i <-> dims[i]); 0 -> 8   */
  int ssim_step[CZC_MAX_DIMS];   /* window step per input axis; 0 -> 1 (L352: w = 8, step 1)     */
  int ssim_range_mode;           /* 0: L = max - min of the original window (reading R15)        */
                                 /* 1: L = value range of the whole original field               */
  int ac_max_lag;                /* autocorrelation lags 1..ac_max_lag (<= CZC_MAX_LAG); 0 -> 10 */
  int timing;                    /* 1: record per-pattern device time into czc_result.kernel_ms  */
  int rank, nranks;              /* slab mode over nranks GPUs; nranks <= 1: single GPU          */
  const void* nccl_uid;          /* 128-byte ncclUniqueId (from rank 0), required if nranks > 1; */
                                 /* given with nranks = 1 it runs the NCCL slab path on 1 rank  */
  double* debug_wssim;           /* optional DEVICE buffer of n_windows doubles: local SSIM of   */
                                 /* every window in C order of the window-origin grid (Alg. 3    */
                                 /* L310 "wssim"); NULL = not written (not on the timed path)    */
  int loopback_slabs;            /* verification of slab mode on ONE GPU: > 1 splits dims[0]    */
                                 /* into that many slabs and runs the exact multi-GPU path (halo */
                                 /* buffers, owned ranges, rank-ordered combine) with device     */
                                 /* copies in place of NCCL; 0/1 = off.  Requires nranks <= 1.   */
  int pdf_bins;                  /* CZC_M_PDF: bins per PDF, 1..CZC_PDF_MAX_BINS; 0 -> 100       */
  double* debug_der;             /* optional DEVICE buffer of 5 x n_interior doubles: the error   */
                                 /* dF = F(recon) - F(orig) of every interior point (Alg. 2 */
                                 /* "Der"), field-major (DER1, DER2, GRAD, DIV, LAP), points in C  */
                                 /* order of the interior grid (extent n_a - 2 per active axis);  */
                                 /* NULL = not written (not on the timed path)                    */
} czc_config;

/* Field shape.  Single GPU: z0 = 0 and nz_local = dims[0] (or 0 meaning dims[0]).
 * Slab mode: dims are GLOBAL; this rank's buffers hold planes [z0, z0 + nz_local) of axis 0. */
typedef struct czc_shape {
  int ndim;
  int64_t dims[CZC_MAX_DIMS];
  int64_t z0;
  int64_t nz_local;
} czc_shape;

typedef struct czc_deriv_stats {  /* statistics of dF = F(recon) - F(orig) over interior points */
  double maxabs, mae, mse, rmse;  /* max |dF|, mean |dF|, mean dF^2, sqrt(mse)                  */
  double f_min, f_max;            /* extrema of F(orig)                                          */
  double psnr;                    /* 20 log10(f_max - f_min) - 10 log10(mse)                     */
} czc_deriv_stats;

typedef struct czc_result {
  uint64_t computed_mask;        /* groups actually computed (subset of the requested mask)      */
  /* ---- P1 (Table I Category I, L107; north_star list) ---------------------------------------- */
  uint64_t n;
  double x_min, x_max, value_range;                   /* of the original; R = x_max - x_min     */
  double err_min, err_max, err_maxabs;                /* e = recon - orig (signed), max |e|      */
  double err_mean, err_absmean;
  double mse, rmse, nrmse, psnr, snr, max_rel_err;    /* nrmse = rmse/R, max_rel_err = max|e|/R  */
  double pwr_min, pwr_max, pwr_mean;                  /* point-wise |e|/|x| over x != 0          */
  uint64_t n_pwr;
  double pearson, err_var;
  /* ---- P2 derivatives (Eq. 1) ----------------------------------------------------- */
  uint64_t n_interior;
  czc_deriv_stats deriv[CZC_NDERIV];                  /* DER1, DER2, GRAD, DIV, LAP              */
  /* ---- P2 autocorrelation (Eq. 2) ------------------------------------------------------- */
  int32_t ac_max_lag, _pad0;
  double ac[CZC_MAX_LAG + 1];                         /* ac[0] = 1                               */
  uint64_t ac_count[CZC_MAX_LAG + 1];                 /* ne_tau = prod_a (n_a - tau)             */
  /* ---- P3 SSIM (L139-L146) ------------------------------------------------------------------- */
  int32_t ssim_window[CZC_MAX_DIMS], ssim_step[CZC_MAX_DIMS];   /* as used, per input axis      */
  uint64_t n_windows;
  double ssim;
  uint64_t n_ssim_exact;         /* windows whose fast-path error bound failed and were          */
                                 /* recomputed by the exact per-window path                      */
  /* ---- PDFs (Table I Category I "Error PDF", "Pwr error PDF"; reading R24) ------ */
  /* pdf_bins equal-width bins over [lo, lo + pdf_bins * width]: the error e over [err_min,        */
  /* err_max] (all N elements), the point-wise relative error |e|/|x| over [pwr_min, pwr_max]      */
  /* (elements with x != 0).  Bin of v: floor((v - lo) / width) in IEEE double, the top edge       */
  /* clamped into the last bin; width 0 (all values equal) puts everything in bin 0.  Counts are   */
  /* exact integers; the density of bin b is count[b] / (total * width).                          */
  int32_t pdf_bins, _pad1;
  double err_pdf_lo, err_pdf_width, pwr_pdf_lo, pwr_pdf_width;
  uint64_t err_pdf[CZC_PDF_MAX_BINS];
  uint64_t pwr_pdf[CZC_PDF_MAX_BINS];
  /* ---- timing (cfg.timing) ------------------------------------------------------------------- */
  float kernel_ms[6];            /* device ms on the context stream: P1, P2 derivatives, P2      */
                                 /* autocorrelation, P3 SSIM, whole call, (reserved = 0)         */
} czc_result;

typedef struct czc_ctx czc_ctx;

/* Create a context bound to cfg->device (NULL cfg = defaults).  In slab mode (nranks > 1) this
 * also creates the NCCL communicator (collective across ranks: every rank must call it).
 * *ctx is owned by the caller and released with czc_free. */
czc_status czc_init(czc_ctx** ctx, const czc_config* cfg);

/* Assess a field pair resident in DEVICE memory.
 *   orig, recon : caller-owned device pointers to shape->nz_local * dims[1] * dims[2] elements of
 *                 `dtype` (read-only; element-aligned; 16-byte alignment takes the vector path).
 *   dtype       : CZC_F32 or CZC_F64 (both fields), else CZC_ERR_DTYPE.
 *   metric_mask : OR of CZC_M_* bits; groups run in the order P1 -> P2 -> P3 (AC needs P1's
 *                 mean and variance of the error, Alg. 2).
 *   out         : caller-owned host struct, filled before return.
 * Slab mode: collective — every rank calls with its own slab; all ranks receive identical *out. */
czc_status czc_assess(czc_ctx* ctx, const void* orig, const void* recon, const czc_shape* shape,
                      czc_dtype dtype, uint64_t metric_mask, czc_result* out);

/* Same as czc_assess, but orig/recon are HOST pointers: the library copies them into
 * context-owned device buffers on its stream (pinned host memory gives full PCIe/C2C speed),
 * then runs the same kernels.  Used for end-to-end measurement. */
czc_status czc_assess_host(czc_ctx* ctx, const void* orig, const void* recon, const czc_shape* shape,
                           czc_dtype dtype, uint64_t metric_mask, czc_result* out);

/* Rank-ordered combine of per-slab partial records and the metric finish — the host step of slab
 * mode, exported so it can be verified without a GPU.  `records` holds `nrecords` consecutive
 * records of czc_sizeof(3) bytes each (slab order = rank order), `global_shape` the whole field
 * (z0 = 0, nz_local = 0), `cfg` the SSIM / AC settings used to produce them.  Host memory only. */
czc_status czc_combine(const void* records, int nrecords, const czc_shape* global_shape,
                       const czc_config* cfg, uint64_t metric_mask, czc_result* out);

/* Release the context, its device scratch, its stream (if owned) and its NCCL communicator. */
void czc_free(czc_ctx* ctx);

/* Static human-readable string for a status; never NULL. */
const char* czc_strerror(czc_status status);

/* Last error detail recorded in ctx (e.g. the CUDA error string); never NULL. */
const char* czc_last_error(const czc_ctx* ctx);

/* ABI version (CZC_ABI_VERSION) and whether NCCL slab mode was compiled in (1/0). */
int czc_abi_version(void);
int czc_has_nccl(void);

/* sizeof(czc_config) (what = 0), sizeof(czc_shape) (1), sizeof(czc_result) (2), size of one
 * partial record (3: what czc_combine consumes per slab), bytes of a record copied device->host
 * when no PDF is requested (4: one record per single-GPU czc_assess call, one per slab / z-chunk
 * in slab mode and czc_assess_host); 0 otherwise.  Lets bindings verify their struct mirrors
 * against the compiled library. */
uint64_t czc_sizeof(int what);

#ifdef __cplusplus
}
#endif
#endif /* CZC_H */

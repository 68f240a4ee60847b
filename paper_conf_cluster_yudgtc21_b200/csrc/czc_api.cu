// czc_api.cu — the C ABI (include/czc.h): context, validation, the "GPU module coordinator"
// (L96: identify the requested metric categories, launch the matching fused kernels), the slab
// decomposition for several GPUs (L423 future work), one device->host copy of
// the partial records, and the scalar finish math (derived metrics).
#include <cuda_runtime.h>
#include <math.h>
#include <stddef.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <new>
#include <string>
#include <utility>
#include <vector>

#include <nvtx3/nvToolsExt.h>   // header-only NVTX 3: host ranges for nsys / ncu --nvtx (no-ops without a tool)

#include "czc_comm.h"
#include "czc_internal.cuh"

// Host-side NVTX range for the duration of a scope (tracing: `ncu --nvtx --nvtx-include czc/`).
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

namespace czc {
// Launchers, instantiated for E = float and E = double in their .cu files.
template <typename E>
cudaError_t launch_p1(const E* x, const E* y, int64_t n, int grid_cap, P1State* parts,
                      DevResults* res, unsigned int* ticket, cudaStream_t st);
cudaError_t launch_p1_combine(const P1State* states, int count, DevResults* res, cudaStream_t st);
template <typename E>
cudaError_t launch_pdf(const E* x, const E* y, int64_t n, int nb, int grid_cap, DevResults* res,
                       cudaStream_t st);
int p1_max_blocks_per_sm();
template <typename E>
int64_t deriv_blocks(const Field3<E>& s, int zchunk);
template <typename E>
int64_t ac_blocks(const Field3<E>& s, int T);
template <typename E>
cudaError_t launch_deriv(const Field3<E>& s, int zchunk, double* parts, DevResults* res,
                         unsigned int* ticket, double* dbg, cudaStream_t st);
template <typename E>
cudaError_t launch_ac(const Field3<E>& s, int T, int zchunk, double* parts, DevResults* res,
                      unsigned int* ticket, cudaStream_t st);
template <typename E>
cudaError_t launch_ssim(int kind, int W, const Field3<E>& f, const SsimParams& p,
                        double* parts, DevResults* res, unsigned int* ticket, double* dbg,
                        cudaStream_t st, int64_t* nblocks_out);
// 4-D fields (p4_generic.cu)
int64_t g4_max_blocks(int sms);
template <typename E>
cudaError_t launch_deriv4(const E* x, const E* y, const int64_t n[4], int sms, double* parts, DevResults* res,
                          unsigned int* ticket, double* dbg, cudaStream_t st);
template <typename E>
cudaError_t launch_ac4(const E* x, const E* y, const int64_t n[4], int T, int sms, double* parts, DevResults* res,
                       unsigned int* ticket, cudaStream_t st);
template <typename E>
cudaError_t launch_ssim4(const E* x, const E* y, const int64_t n[4], const int w[4], const int stp[4], int range_mode,
                         int sms, double* parts, DevResults* res, unsigned int* ticket, double* dbg, cudaStream_t st);
}  // namespace czc

using namespace czc;

static constexpr int kMaxHostChunks = 16;   // z-chunks of the pipelined czc_assess_host
static constexpr int kHostChunks = 8;       // default chunk count

struct czc_ctx {
  czc_config cfg;
  int device = 0;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  int sm_count = 0;
  int p1_grid_cap = 0;
  DevResults* dres = nullptr;      // device
  Record* hrec = nullptr;          // pinned host, max_records records
  unsigned int* tickets = nullptr; // device
  void* parts = nullptr;           // per-block partial records: one region per kernel kind
  size_t parts_cap = 0;
  size_t off_deriv = 0, off_ac = 0, off_ssim = 0;   // byte offsets (P1 at 0) set by ensure_scratch
  // the single-GPU sequence as two concurrent branches (P1 -> AC | derivatives -> SSIM)
  cudaStream_t stream2 = nullptr, stream3 = nullptr;
  cudaEvent_t fork_ev = nullptr, join_ev = nullptr, join3_ev = nullptr, p1_ev = nullptr;
  bool concurrent = true;          // CZC_SEQUENTIAL=1: one stream (A/B timing)
  int layout = 0;                  // CZC_BRANCHES (A/B): 0 P1>AC | deriv>SSIM, 1 P1>AC>deriv | SSIM, 2 P1>AC | deriv | SSIM
  void* din[2] = {nullptr, nullptr};    // staging for czc_assess_host
  size_t din_cap = 0;
  cudaEvent_t ev[6] = {};   // P1 start, P1 end, deriv end, AC end, SSIM end, call end
  std::string last_error;
  // slab mode (NCCL ranks or loopback)
  CommState* comm = nullptr;
  void* dgather_in = nullptr;      // device, 64 B
  void* dgather = nullptr;         // device, max_records * sizeof(Record)
  void* dstates = nullptr;         // device, max_records * sizeof(P1State)
  void* halo = nullptr;            // device halo planes (x lo, y lo, x hi, y hi)
  size_t halo_cap = 0;
  int max_records = 1;
  // single-GPU launch sequence replayed as one CUDA graph while the call signature repeats
  cudaGraphExec_t gexec = nullptr;
  std::vector<int64_t> gkey;
  bool use_graphs = true;          // CZC_NO_GRAPHS=1 disables (A/B timing)
  // pipelined host path
  cudaStream_t copy_stream[2] = {nullptr, nullptr};   // [0]: H2D chunks (x then y); [1] unused
  cudaEvent_t copy_ev[2][kMaxHostChunks] = {};
  // NCCL slab mode: halo exchange on its own stream (overlapping P1), and the validated slab
  // table of the last call signature (re-validated collectively only when the signature changes)
  cudaStream_t halo_stream = nullptr;
  cudaEvent_t halo_ev[2] = {};        // [0]: inputs ready on the compute stream, [1]: halos received
  std::vector<int64_t> slab_key;
  std::vector<int64_t> slab_tab;      // 2 per rank: z0, nz_local
  int64_t* hpin = nullptr;            // pinned host staging for the small slab-table copies
};

static const char* kStatusStr[] = {"ok", "invalid argument", "invalid shape", "unsupported dtype",
                                   "CUDA error", "out of memory", "communication (NCCL) error",
                                   "unsupported"};

extern "C" const char* czc_strerror(czc_status s) {
  const int i = (int)s;
  return (i >= 0 && i < 8) ? kStatusStr[i] : "unknown status";
}
extern "C" const char* czc_last_error(const czc_ctx* ctx) { return ctx ? ctx->last_error.c_str() : ""; }
extern "C" int czc_abi_version(void) { return CZC_ABI_VERSION; }
extern "C" int czc_has_nccl(void) { return comm_available(); }
extern "C" uint64_t czc_sizeof(int what) {
  return what == 0 ? sizeof(czc_config) : what == 1 ? sizeof(czc_shape) : what == 2 ? sizeof(czc_result)
       : what == 3 ? sizeof(Record) : what == 4 ? kRecordNoPdf : 0;
}

static czc_status cuda_fail(czc_ctx* ctx, cudaError_t e, const char* where) {
  if (ctx) ctx->last_error = std::string(where) + ": " + cudaGetErrorString(e);
  (void)cudaGetLastError();
  return e == cudaErrorMemoryAllocation ? CZC_ERR_NOMEM : CZC_ERR_CUDA;
}
#define CZC_CUDA(ctx, call)                                    \
  do {                                                         \
    cudaError_t _e = (call);                                   \
    if (_e != cudaSuccess) return cuda_fail((ctx), _e, #call); \
  } while (0)

static czc_status validate_config(const czc_config& c) {
  if (c.ac_max_lag < 0 || c.ac_max_lag > CZC_MAX_LAG) return CZC_ERR_INVALID;
  if (c.ssim_range_mode < 0 || c.ssim_range_mode > 1) return CZC_ERR_INVALID;
  for (int i = 0; i < CZC_MAX_DIMS; i++)
    if (c.ssim_window[i] < 0 || c.ssim_step[i] < 0) return CZC_ERR_INVALID;
  if (c.nranks > 1 && (c.rank < 0 || c.rank >= c.nranks || !c.nccl_uid)) return CZC_ERR_INVALID;
  if (c.nccl_uid && (c.nranks < 1 || c.rank < 0 || c.rank >= c.nranks)) return CZC_ERR_INVALID;
  if (c.loopback_slabs < 0 || (c.loopback_slabs > 1 && (c.nranks > 1 || c.nccl_uid))) return CZC_ERR_INVALID;
  if (c.pdf_bins < 0 || c.pdf_bins > CZC_PDF_MAX_BINS) return CZC_ERR_INVALID;
  return CZC_OK;
}

extern "C" czc_status czc_init(czc_ctx** out, const czc_config* cfg) {
  if (!out) return CZC_ERR_INVALID;
  *out = nullptr;
  czc_config c;
  memset(&c, 0, sizeof(c));
  if (cfg) c = *cfg;
  else c.device = -1;
  czc_status st = validate_config(c);
  if (st != CZC_OK) return st;
  const bool slab_mode = c.nranks > 1 || c.nccl_uid != nullptr;   // NCCL comm (also valid with 1 rank)
  if (slab_mode && !comm_available()) return CZC_ERR_UNSUPPORTED;

  czc_ctx* ctx = new (std::nothrow) czc_ctx();
  if (!ctx) return CZC_ERR_NOMEM;
  ctx->cfg = c;
  {
    const char* ng = getenv("CZC_NO_GRAPHS");
    ctx->use_graphs = !(ng && ng[0] == '1');
    const char* sq = getenv("CZC_SEQUENTIAL");
    ctx->concurrent = !(sq && sq[0] == '1');
    const char* br = getenv("CZC_BRANCHES");
    ctx->layout = br ? atoi(br) : 0;
  }
  ctx->max_records = std::max(kMaxHostChunks, std::max(c.nranks, c.loopback_slabs));
  do {
    int dev = c.device;
    if (dev < 0) {
      if (cudaGetDevice(&dev) != cudaSuccess) { st = cuda_fail(ctx, cudaGetLastError(), "cudaGetDevice"); break; }
    }
    ctx->device = dev;
    cudaError_t e = cudaSetDevice(dev);
    if (e != cudaSuccess) { st = cuda_fail(ctx, e, "cudaSetDevice"); break; }
    cudaDeviceGetAttribute(&ctx->sm_count, cudaDevAttrMultiProcessorCount, dev);
    ctx->p1_grid_cap = ctx->sm_count * p1_max_blocks_per_sm();
    if (c.stream) {
      ctx->stream = (cudaStream_t)c.stream;
    } else {
      // a BLOCKING stream: it is ordered after work the caller queued on the legacy default
      // stream (e.g. the kernels that produced the fields), as a NULL stream argument implies
      e = cudaStreamCreateWithFlags(&ctx->stream, cudaStreamDefault);
      if (e != cudaSuccess) { st = cuda_fail(ctx, e, "cudaStreamCreate"); break; }
      ctx->own_stream = true;
    }
    const size_t rb = (size_t)ctx->max_records * sizeof(Record);
    if ((e = cudaMalloc(&ctx->dres, sizeof(DevResults))) != cudaSuccess) { st = cuda_fail(ctx, e, "cudaMalloc(res)"); break; }
    // every record byte is defined (the D2H copy of a call carries slots of groups it did not run)
    if ((e = cudaMemsetAsync(ctx->dres, 0, sizeof(DevResults), ctx->stream)) != cudaSuccess) { st = cuda_fail(ctx, e, "cudaMemset(res)"); break; }
    if ((e = cudaMallocHost(&ctx->hrec, rb)) != cudaSuccess) { st = cuda_fail(ctx, e, "cudaMallocHost"); break; }
    if ((e = cudaMallocHost(&ctx->hpin, (size_t)(4 + 3 * ctx->max_records) * sizeof(int64_t))) != cudaSuccess) {
      st = cuda_fail(ctx, e, "cudaMallocHost");
      break;
    }
    if ((e = cudaMalloc(&ctx->tickets, TICKET_N * sizeof(unsigned int))) != cudaSuccess) { st = cuda_fail(ctx, e, "cudaMalloc(tickets)"); break; }
    if ((e = cudaMemsetAsync(ctx->tickets, 0, TICKET_N * sizeof(unsigned int), ctx->stream)) != cudaSuccess ||
        (e = cudaStreamSynchronize(ctx->stream)) != cudaSuccess) { st = cuda_fail(ctx, e, "cudaMemset"); break; }
    for (int i = 0; i < 6 && st == CZC_OK; i++)
      if ((e = cudaEventCreate(&ctx->ev[i])) != cudaSuccess) st = cuda_fail(ctx, e, "cudaEventCreate");
    if (st != CZC_OK) break;
    if ((e = cudaStreamCreateWithFlags(&ctx->stream2, cudaStreamNonBlocking)) != cudaSuccess ||
        (e = cudaStreamCreateWithFlags(&ctx->stream3, cudaStreamNonBlocking)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&ctx->join3_ev, cudaEventDisableTiming)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&ctx->fork_ev, cudaEventDisableTiming)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&ctx->join_ev, cudaEventDisableTiming)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&ctx->p1_ev, cudaEventDisableTiming)) != cudaSuccess) {
      st = cuda_fail(ctx, e, "second stream");
      break;
    }
    {
      if ((e = cudaMalloc(&ctx->dgather_in, 64)) != cudaSuccess) { st = cuda_fail(ctx, e, "cudaMalloc(gather)"); break; }
      if ((e = cudaMalloc(&ctx->dgather, rb)) != cudaSuccess) { st = cuda_fail(ctx, e, "cudaMalloc(gather)"); break; }
      if ((e = cudaMalloc(&ctx->dstates, (size_t)ctx->max_records * sizeof(P1State))) != cudaSuccess) { st = cuda_fail(ctx, e, "cudaMalloc(states)"); break; }
    }
    if (slab_mode) {
      if ((e = cudaStreamCreateWithFlags(&ctx->halo_stream, cudaStreamNonBlocking)) != cudaSuccess ||
          (e = cudaEventCreateWithFlags(&ctx->halo_ev[0], cudaEventDisableTiming)) != cudaSuccess ||
          (e = cudaEventCreateWithFlags(&ctx->halo_ev[1], cudaEventDisableTiming)) != cudaSuccess) {
        st = cuda_fail(ctx, e, "halo stream");
        break;
      }
      ctx->comm = comm_create(c.nccl_uid, c.rank, std::max(1, c.nranks), &ctx->last_error);
      if (!ctx->comm) { st = CZC_ERR_COMM; break; }
    }
  } while (0);
  if (st != CZC_OK) {
    czc_free(ctx);
    return st;
  }
  *out = ctx;
  return CZC_OK;
}

extern "C" void czc_free(czc_ctx* ctx) {
  if (!ctx) return;
  cudaSetDevice(ctx->device);
  if (ctx->stream) cudaStreamSynchronize(ctx->stream);
  if (ctx->comm) comm_destroy(ctx->comm);
  cudaFree(ctx->dres);
  cudaFreeHost(ctx->hrec);
  cudaFreeHost(ctx->hpin);
  cudaFree(ctx->tickets);
  cudaFree(ctx->parts);
  cudaFree(ctx->din[0]);
  cudaFree(ctx->din[1]);
  cudaFree(ctx->dgather_in);
  cudaFree(ctx->dgather);
  cudaFree(ctx->dstates);
  cudaFree(ctx->halo);
  for (int i = 0; i < 6; i++)
    if (ctx->ev[i]) cudaEventDestroy(ctx->ev[i]);
  for (int c = 0; c < 2; c++) {
    for (int i = 0; i < kMaxHostChunks; i++)
      if (ctx->copy_ev[c][i]) cudaEventDestroy(ctx->copy_ev[c][i]);
    if (ctx->copy_stream[c]) cudaStreamDestroy(ctx->copy_stream[c]);
  }
  if (ctx->gexec) cudaGraphExecDestroy(ctx->gexec);
  for (cudaStream_t sx : {ctx->stream2, ctx->stream3})
    if (sx) { cudaStreamSynchronize(sx); cudaStreamDestroy(sx); }
  for (cudaEvent_t ev : {ctx->fork_ev, ctx->join_ev, ctx->join3_ev, ctx->p1_ev})
    if (ev) cudaEventDestroy(ev);
  for (int i = 0; i < 2; i++)
    if (ctx->halo_ev[i]) cudaEventDestroy(ctx->halo_ev[i]);
  if (ctx->halo_stream) cudaStreamDestroy(ctx->halo_stream);
  if (ctx->own_stream && ctx->stream) cudaStreamDestroy(ctx->stream);
  delete ctx;
}

// ------------------------------------------------------------------------------------------------
// Planning (global shape; host only)
// ------------------------------------------------------------------------------------------------
namespace {
struct Plan {
  int64_t g3[3] = {1, 1, 1};      // GLOBAL field, extent-1 axes squeezed, right-aligned (nz, ny, nx)
  int64_t g4[4] = {1, 1, 1, 1};   // the same right-aligned into four axes (D = 4: all active)
  int D = 0;                      // active axes
  int win4[4] = {1, 1, 1, 1}, step4[4] = {1, 1, 1, 1};   // SSIM per right-aligned axis (D = 4)
  int W = 8, step[3] = {1, 1, 1}; // SSIM (per 3-D axis)
  int win3[3] = {1, 1, 1};
  int kind = 0;                   // 3, 2, 1 (active axes of the SSIM window)
  int T = 10;
  int nb = 100;                   // PDF bins
  bool run_p1 = false, run_deriv = false, run_ac = false, run_ssim = false, run_pdf = false;
  int32_t win_in[4] = {0, 0, 0, 0}, step_in[4] = {0, 0, 0, 0};  // reported per input axis
};

czc_status make_plan(const czc_config& c, int ndim, const int64_t* dims, uint64_t mask, Plan& P, std::string& why) {
  if (ndim < 1 || ndim > CZC_MAX_DIMS) { why = "ndim must be 1..4"; return CZC_ERR_SHAPE; }
  int64_t gd[CZC_MAX_DIMS];
  for (int i = 0; i < ndim; i++) {
    if (dims[i] < 1) { why = "dims must be >= 1"; return CZC_ERR_SHAPE; }
    gd[i] = dims[i];
  }
  // squeeze inactive (extent-1) axes; the C-order layout is unchanged by it
  int act_in[CZC_MAX_DIMS], na = 0;
  for (int i = 0; i < ndim; i++)
    if (gd[i] > 1) act_in[na++] = i;
  P.D = na;
  for (int k = 0; k < na; k++) P.g4[4 - na + k] = gd[act_in[k]];
  if (na <= 3)
    for (int k = 0; k < na; k++) P.g3[3 - na + k] = gd[act_in[k]];
  P.T = c.ac_max_lag ? c.ac_max_lag : 10;
  P.run_ssim = (mask & CZC_M_SSIM) != 0;
  P.run_deriv = (mask & CZC_M_DERIV) != 0;
  P.run_ac = (mask & CZC_M_AUTOCORR) != 0;
  P.run_pdf = (mask & CZC_M_PDF) != 0;
  P.nb = c.pdf_bins ? c.pdf_bins : 100;
  P.run_p1 = (mask & (CZC_M_P1 | CZC_M_AUTOCORR | CZC_M_PDF)) != 0 || (P.run_ssim && c.ssim_range_mode == 1);
  for (int i = 0; i < ndim; i++) {
    const int w = c.ssim_window[i] ? c.ssim_window[i] : 8;
    const int s = c.ssim_step[i] ? c.ssim_step[i] : 1;
    P.win_in[i] = gd[i] > 1 ? w : 1;
    P.step_in[i] = gd[i] > 1 ? s : 1;
  }
  if (P.run_ssim) {
    if (na == 0) { why = "SSIM needs at least one axis with extent > 1"; return CZC_ERR_SHAPE; }
    int W = -1;
    for (int k = 0; k < na; k++) {
      const int w = P.win_in[act_in[k]];
      if (W < 0) W = w;
      if (w != W) { why = "SSIM fast path needs the same window extent on every active axis"; return CZC_ERR_UNSUPPORTED; }
      if (w > gd[act_in[k]]) { why = "SSIM window larger than the field"; return CZC_ERR_SHAPE; }
      P.win4[4 - na + k] = w;
      P.step4[4 - na + k] = P.step_in[act_in[k]];
      if (na <= 3) {
        P.win3[3 - na + k] = w;
        P.step[3 - na + k] = P.step_in[act_in[k]];
      }
    }
    if (W < 2 || W > kMaxWin) { why = "SSIM window extent must be 2..16"; return CZC_ERR_UNSUPPORTED; }
    P.W = W;
    P.kind = na;
  }
  return CZC_OK;
}

inline double nan_() { return NAN; }

void finish_p1(const P1State& f, czc_result* o) {
  const double n = f.n;
  o->n = (uint64_t)n;
  o->x_min = f.xmin;
  o->x_max = f.xmax;
  const double R = (double)f.xmax - (double)f.xmin;
  o->value_range = R;
  o->err_min = f.emin;
  o->err_max = f.emax;
  o->err_maxabs = fmax(fabs(f.emin), fabs(f.emax));
  o->err_mean = f.me;
  o->err_absmean = f.sae / n;
  const double se2 = f.m2e + n * f.me * f.me;     // sum e^2 (positive terms)
  const double mse = se2 / n;
  o->mse = mse;
  o->rmse = sqrt(mse);
  o->nrmse = R > 0 ? sqrt(mse) / R : (mse > 0 ? INFINITY : nan_());
  o->psnr = mse == 0 ? INFINITY : (R == 0 ? -INFINITY : 20.0 * log10(R) - 10.0 * log10(mse));
  o->snr = se2 == 0 ? (f.m2x > 0 ? INFINITY : nan_()) : 10.0 * log10(f.m2x / se2);
  o->max_rel_err = R > 0 ? o->err_maxabs / R : (o->err_maxabs > 0 ? INFINITY : nan_());
  o->n_pwr = (uint64_t)f.npwr;
  o->pwr_min = f.npwr > 0 ? f.pmin : nan_();
  o->pwr_max = f.npwr > 0 ? f.pmax : nan_();
  o->pwr_mean = f.npwr > 0 ? f.spwr / f.npwr : nan_();
  o->pearson = (f.m2x > 0 && f.m2y > 0) ? f.cxy / sqrt(f.m2x * f.m2y) : nan_();
  o->err_var = f.m2e / n;
}

// Rank-ordered combine of records (P1 states by the stable pairwise merge, sums added, extrema
// min/max), then the derived metrics from the global shape in P.g3.  Host code; every rank runs
// it on the same bytes, so all ranks return identical results.
void combine_and_finish(const Plan& P, const Record* recs, int nrec, uint64_t mask, czc_result* out) {
  Record R = recs[0];
  P1State g;
  p1_empty(g);
  for (int r = 0; r < nrec; r++) p1_merge(g, recs[r].p1);
  R.p1 = g;
  for (int r = 1; r < nrec; r++) {
    for (int k = 0; k < kDerivSlots; k++) {
      const int op = deriv_op(k);
      R.deriv[k] = op == OP_SUM ? R.deriv[k] + recs[r].deriv[k]
                 : op == OP_MIN ? std::min(R.deriv[k], recs[r].deriv[k]) : std::max(R.deriv[k], recs[r].deriv[k]);
    }
    for (int w = 0; w < kAcWalks; w++)
      for (int k = 0; k < kAcSlots; k++) R.ac[w][k] += recs[r].ac[w][k];
    for (int k = 0; k < kSsimSlots; k++) R.ssim[k] += recs[r].ssim[k];
    if (P.run_pdf)
      for (int h = 0; h < 2; h++)
        for (int b = 0; b < P.nb; b++) R.pdf[h][b] += recs[r].pdf[h][b];
  }
  uint64_t done = 0;
  if (P.run_p1 && (mask & CZC_M_P1)) { finish_p1(R.p1, out); done |= CZC_M_P1; }
  if (P.run_deriv) {
    int64_t nI = P.D > 0 ? 1 : 0;
    for (int a = 0; a < 4; a++)
      if (P.g4[a] > 1) nI *= std::max<int64_t>(P.g4[a] - 2, 0);
    out->n_interior = (uint64_t)nI;
    for (int f = 0; f < CZC_NDERIV; f++) {
      const double* r = R.deriv + f * kDerivStats;
      czc_deriv_stats& d = out->deriv[f];
      if (nI == 0) {
        d.maxabs = d.mae = d.mse = d.rmse = d.f_min = d.f_max = d.psnr = NAN;
        continue;
      }
      d.maxabs = r[0];
      d.mae = r[1] / (double)nI;
      d.mse = r[2] / (double)nI;
      d.rmse = sqrt(d.mse);
      d.f_min = r[3];
      d.f_max = r[4];
      const double rng = d.f_max - d.f_min;
      d.psnr = d.mse == 0 ? INFINITY : (rng == 0 ? -INFINITY : 20.0 * log10(rng) - 10.0 * log10(d.mse));
    }
    done |= CZC_M_DERIV;
  }
  if (P.run_ac) {
    out->ac_max_lag = P.T;
    const double var = R.p1.m2e / R.p1.n;
    int64_t nmin = INT64_MAX;
    for (int a = 0; a < 4; a++)
      if (P.g4[a] > 1) nmin = std::min(nmin, P.g4[a]);
    out->ac[0] = 1.0;
    out->ac_count[0] = (uint64_t)(P.g4[0] * P.g4[1] * P.g4[2] * P.g4[3]);
    for (int t = 1; t <= CZC_MAX_LAG; t++) {
      if (t > P.T || P.D == 0 || t >= nmin) { out->ac[t] = NAN; out->ac_count[t] = 0; continue; }
      int64_t ne = 1;
      for (int a = 0; a < 4; a++) ne *= P.g4[a] > 1 ? P.g4[a] - t : 1;
      out->ac_count[t] = (uint64_t)ne;
      const double S = R.ac[0][t - 1] + R.ac[1][t - 1] + R.ac[2][t - 1];   // z, y, x walks
      out->ac[t] = var > 0 ? S / (double)P.D / (double)ne / var : NAN;
    }
    done |= CZC_M_AUTOCORR;
  }
  if (P.run_ssim) {
    for (int i = 0; i < CZC_MAX_DIMS; i++) { out->ssim_window[i] = P.win_in[i]; out->ssim_step[i] = P.step_in[i]; }
    out->n_windows = (uint64_t)R.ssim[1];
    out->ssim = R.ssim[1] > 0 ? R.ssim[0] / R.ssim[1] : NAN;
    out->n_ssim_exact = (uint64_t)R.ssim[2];
    done |= CZC_M_SSIM;
  }
  if (P.run_pdf) {
    // the ranges are the global P1 extrema, computed exactly as on the device (pdf_range)
    const PdfRange re = pdf_range(R.p1.emin, R.p1.emax, P.nb);
    const PdfRange rp = pdf_range(R.p1.pmin, R.p1.pmax, P.nb);
    out->pdf_bins = P.nb;
    out->err_pdf_lo = re.lo;
    out->err_pdf_width = re.w;
    out->pwr_pdf_lo = R.p1.npwr > 0 ? rp.lo : NAN;
    out->pwr_pdf_width = R.p1.npwr > 0 ? rp.w : NAN;
    for (int b = 0; b < P.nb; b++) { out->err_pdf[b] = R.pdf[0][b]; out->pwr_pdf[b] = R.pdf[1][b]; }
    done |= CZC_M_PDF;
  }
  out->computed_mask = done;
}
}  // namespace

extern "C" czc_status czc_combine(const void* records, int nrecords, const czc_shape* global_shape,
                                  const czc_config* cfg, uint64_t metric_mask, czc_result* out) {
  if (!out) return CZC_ERR_INVALID;
  memset(out, 0, sizeof(*out));
  if (!records || nrecords < 1 || !global_shape || !cfg) return CZC_ERR_INVALID;
  czc_status st = validate_config(*cfg);
  if (st != CZC_OK) return st;
  Plan P;
  std::string why;
  st = make_plan(*cfg, global_shape->ndim, global_shape->dims, metric_mask, P, why);
  if (st != CZC_OK) return st;
  std::vector<Record> recs(nrecords);
  memcpy(recs.data(), records, (size_t)nrecords * sizeof(Record));
  combine_and_finish(P, recs.data(), nrecords, metric_mask, out);
  return CZC_OK;
}

// ------------------------------------------------------------------------------------------------
// Device execution
// ------------------------------------------------------------------------------------------------
// Grow a context buffer.  Work already queued on the context stream may still use the old
// buffer (e.g. P1's partials when the P2/P3 scratch grows), so the stream is drained before the
// free: cudaFree does not order itself after work on a non-blocking stream.
static czc_status ensure_buf(czc_ctx* ctx, void** p, size_t* cap, size_t bytes) {
  if (bytes <= *cap) return CZC_OK;
  if (*p) CZC_CUDA(ctx, cudaStreamSynchronize(ctx->stream));
  cudaFree(*p);
  *p = nullptr;
  *cap = 0;
  CZC_CUDA(ctx, cudaMalloc(p, bytes));
  *cap = bytes;
  return CZC_OK;
}

namespace {
constexpr int kZchunkDeriv = 128, kZchunkSsim = 32;

SsimParams ssim_params(const Plan& P, const czc_config& c) {
  SsimParams sp{};
  sp.sz = P.step[0]; sp.sy = P.step[1]; sp.sx = P.step[2];
  sp.zchunk = kZchunkSsim;
  sp.range_mode = c.ssim_range_mode;
  sp.nwz = (P.g3[0] - P.win3[0]) / sp.sz + 1;
  sp.nwy = (P.g3[1] - P.win3[1]) / sp.sy + 1;
  sp.nwx = (P.g3[2] - P.win3[2]) / sp.sx + 1;
  return sp;
}

// halo depth above a slab: derivatives need 1 plane, AC T planes, SSIM W - 1 planes
int64_t halo_depth(const Plan& P) {
  int64_t H = 0;
  if (P.run_deriv) H = std::max<int64_t>(H, 1);
  if (P.run_ac) H = std::max<int64_t>(H, P.T);
  if (P.run_ssim) H = std::max<int64_t>(H, P.W - 1);
  return H;
}
}  // namespace

// Scratch for every launch over the given field view: one region per kernel kind (P1 at offset
// 0, then derivatives, AC, SSIM), so kernels of different kinds may run concurrently.
template <typename E>
static czc_status ensure_scratch(czc_ctx* ctx, const Plan& P, const Field3<E>& F, const SsimParams& sp) {
  auto al = [](size_t b) { return (b + 255) / 256 * 256; };
  const size_t p1 = al((size_t)ctx->p1_grid_cap * sizeof(P1State));
  const size_t dv = P.run_deriv ? al((size_t)deriv_blocks(F, kZchunkDeriv) * kDerivSlots * sizeof(double)) : 0;
  const size_t ac = P.run_ac ? al((size_t)ac_blocks(F, P.T) * kAcSlots * sizeof(double)) : 0;
  size_t ss = 0;
  if (P.run_ssim) {
    int64_t nb = 0;
    if (launch_ssim(P.kind, P.W, F, sp, nullptr, nullptr, nullptr, nullptr, ctx->stream, &nb) != cudaSuccess) {
      ctx->last_error = "unsupported SSIM window";
      return CZC_ERR_UNSUPPORTED;
    }
    ss = al((size_t)nb * kSsimSlots * sizeof(double));
  }
  czc_status st = ensure_buf(ctx, &ctx->parts, &ctx->parts_cap, p1 + dv + ac + ss);
  if (st != CZC_OK) return st;
  ctx->off_deriv = p1;
  ctx->off_ac = p1 + dv;
  ctx->off_ssim = p1 + dv + ac;
  return CZC_OK;
}
static double* parts_at(czc_ctx* ctx, size_t off) { return reinterpret_cast<double*>(static_cast<char*>(ctx->parts) + off); }

// The kernels of P2 / P3 over one field view (the owned planes of F); results land in dres->rec.
template <typename E>
static czc_status launch_deriv_k(czc_ctx* ctx, const Field3<E>& F, cudaStream_t s) {
  NvtxRange r_("czc/P2 derivatives");
  CZC_CUDA(ctx, launch_deriv(F, kZchunkDeriv, parts_at(ctx, ctx->off_deriv), ctx->dres, ctx->tickets + TICKET_DERIV,
                             ctx->cfg.debug_der, s));
  return CZC_OK;
}
template <typename E>
static czc_status launch_ac_k(czc_ctx* ctx, const Plan& P, const Field3<E>& F, cudaStream_t s) {
  NvtxRange r_("czc/P2 autocorrelation");
  CZC_CUDA(ctx, launch_ac(F, P.T, 0, parts_at(ctx, ctx->off_ac), ctx->dres, ctx->tickets + TICKET_ACZ, s));
  return CZC_OK;
}
template <typename E>
static czc_status launch_ssim_k(czc_ctx* ctx, const Plan& P, const Field3<E>& F, const SsimParams& sp, cudaStream_t s) {
  NvtxRange r_("czc/P3 SSIM");
  CZC_CUDA(ctx, launch_ssim(P.kind, P.W, F, sp, parts_at(ctx, ctx->off_ssim), ctx->dres, ctx->tickets + TICKET_SSIM,
                            ctx->cfg.debug_wssim, s, nullptr));
  return CZC_OK;
}

// P2 + P3 in sequence on the context stream.
template <typename E>
static czc_status run_p23(czc_ctx* ctx, const Plan& P, const Field3<E>& F, const SsimParams& sp) {
  const cudaStream_t s = ctx->stream;
  czc_status st = ensure_scratch(ctx, P, F, sp);
  if (st != CZC_OK) return st;
  if (P.run_deriv && (st = launch_deriv_k(ctx, F, s)) != CZC_OK) return st;
  if (ctx->cfg.timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[2], s));
  if (P.run_ac && (st = launch_ac_k(ctx, P, F, s)) != CZC_OK) return st;
  if (ctx->cfg.timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[3], s));
  if (P.run_ssim && (st = launch_ssim_k(ctx, P, F, sp, s)) != CZC_OK) return st;
  return CZC_OK;
}

// D2H copy of n consecutive records; without PDFs only the first kRecordNoPdf bytes of each
// (one strided copy).
static cudaError_t copy_records(Record* h, const Record* d, int n, bool pdf, cudaStream_t s) {
  if (pdf) return cudaMemcpyAsync(h, d, (size_t)n * sizeof(Record), cudaMemcpyDeviceToHost, s);
  return cudaMemcpy2DAsync(h, sizeof(Record), d, sizeof(Record), kRecordNoPdf, (size_t)n,
                           cudaMemcpyDeviceToHost, s);
}

template <typename E>
static czc_status p1_local(czc_ctx* ctx, const Plan& P, const E* x, const E* y, int64_t n) {
  if (!P.run_p1) return CZC_OK;
  czc_status st = ensure_buf(ctx, &ctx->parts, &ctx->parts_cap, (size_t)ctx->p1_grid_cap * sizeof(P1State));
  if (st != CZC_OK) return st;
  CZC_CUDA(ctx, launch_p1(x, y, n, ctx->p1_grid_cap, (P1State*)ctx->parts, ctx->dres, ctx->tickets + TICKET_P1, ctx->stream));
  return CZC_OK;
}

static void finish_timing(czc_ctx* ctx, czc_result* out) {
  if (!ctx->cfg.timing) return;
  for (int i = 0; i < 4; i++) cudaEventElapsedTime(&out->kernel_ms[i], ctx->ev[i], ctx->ev[i + 1]);
  cudaEventElapsedTime(&out->kernel_ms[4], ctx->ev[0], ctx->ev[5]);
  out->kernel_ms[5] = 0.f;
}

// The single-GPU launch sequence: P1 (+ PDF), P2, P3, the D2H copy of the record.  Without
// per-kernel timing it runs as two concurrent branches joined before the record copy — the
// context stream: P1 (+ PDF) -> AC (which needs P1's mean / variance of the error, Alg. 2);
// the second stream: derivatives -> SSIM (which needs P1 only for the global range mode) — so
// the memory-latency-bound P1 and the FP64-bound stencil / window kernels can share the SMs.
template <typename E>
static czc_status enqueue_single(czc_ctx* ctx, const Plan& P, const E* x, const E* y, const Field3<E>& F,
                                 const SsimParams& sp) {
  const cudaStream_t s = ctx->stream;
  const bool timing = ctx->cfg.timing != 0;
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[0], s));
  NvtxRange r_("czc/enqueue");
  if (!timing && ctx->concurrent && (P.run_deriv || P.run_ssim)) {
    const int L = ctx->layout;
    const cudaStream_t s2 = ctx->stream2, s3 = ctx->stream3;
    const cudaStream_t sd = L == 1 ? s : s2;            // derivatives
    const cudaStream_t ss = L == 2 ? s3 : s2;           // SSIM
    czc_status st = ensure_scratch(ctx, P, F, sp);
    if (st != CZC_OK) return st;
    CZC_CUDA(ctx, cudaEventRecord(ctx->fork_ev, s));
    CZC_CUDA(ctx, cudaStreamWaitEvent(s2, ctx->fork_ev, 0));
    if (L == 2) CZC_CUDA(ctx, cudaStreamWaitEvent(s3, ctx->fork_ev, 0));
    if (P.run_deriv && sd != s && (st = launch_deriv_k(ctx, F, sd)) != CZC_OK) return st;
    if (P.run_ssim && sp.range_mode == 0 && (st = launch_ssim_k(ctx, P, F, sp, ss)) != CZC_OK) return st;
    if ((st = p1_local(ctx, P, x, y, F.nz * F.ny * F.nx)) != CZC_OK) return st;
    if (P.run_pdf) CZC_CUDA(ctx, launch_pdf(x, y, F.nz * F.ny * F.nx, P.nb, ctx->p1_grid_cap, ctx->dres, s));
    if (P.run_ssim && sp.range_mode != 0) {            // the global range comes from P1
      CZC_CUDA(ctx, cudaEventRecord(ctx->p1_ev, s));
      CZC_CUDA(ctx, cudaStreamWaitEvent(ss, ctx->p1_ev, 0));
      if ((st = launch_ssim_k(ctx, P, F, sp, ss)) != CZC_OK) return st;
    }
    if (P.run_ac && (st = launch_ac_k(ctx, P, F, s)) != CZC_OK) return st;
    if (P.run_deriv && sd == s && (st = launch_deriv_k(ctx, F, s)) != CZC_OK) return st;
    CZC_CUDA(ctx, cudaEventRecord(ctx->join_ev, s2));
    CZC_CUDA(ctx, cudaStreamWaitEvent(s, ctx->join_ev, 0));
    if (L == 2) {
      CZC_CUDA(ctx, cudaEventRecord(ctx->join3_ev, s3));
      CZC_CUDA(ctx, cudaStreamWaitEvent(s, ctx->join3_ev, 0));
    }
    CZC_CUDA(ctx, copy_records(ctx->hrec, &ctx->dres->rec, 1, P.run_pdf, s));
    return CZC_OK;
  }
  czc_status st = p1_local(ctx, P, x, y, F.nz * F.ny * F.nx);
  if (st != CZC_OK) return st;
  if (P.run_pdf) CZC_CUDA(ctx, launch_pdf(x, y, F.nz * F.ny * F.nx, P.nb, ctx->p1_grid_cap, ctx->dres, s));
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[1], s));
  if ((st = run_p23(ctx, P, F, sp)) != CZC_OK) return st;
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[4], s));
  CZC_CUDA(ctx, copy_records(ctx->hrec, &ctx->dres->rec, 1, P.run_pdf, s));
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[5], s));
  return CZC_OK;
}

// Single GPU, whole field resident.  Every buffer is sized first; the launch sequence is then
// captured once into a CUDA graph and replayed for as long as the call signature (pointers,
// shape, element type, plan, debug buffer, scratch buffer) repeats — one graph launch instead of
// ~8 stream operations per call.  With cfg.timing (per-kernel events) or if capture is
// unavailable the sequence is launched directly.
template <typename E>
static czc_status assess_single(czc_ctx* ctx, const Plan& P, const E* x, const E* y, czc_result* out,
                                uint64_t mask) {
  const cudaStream_t s = ctx->stream;
  Field3<E> F{};
  F.nz = P.g3[0]; F.ny = P.g3[1]; F.nx = P.g3[2];
  F.zown0 = 0; F.zown1 = F.nz;
  F.nseg = 1; F.xs[0] = x; F.ys[0] = y; F.zs[0] = 0; F.zs[1] = F.nz;
  const SsimParams sp = ssim_params(P, ctx->cfg);
  czc_status st = ensure_scratch(ctx, P, F, sp);       // no allocation inside the sequence
  if (st != CZC_OK) return st;
  bool launched = false;
  if (ctx->use_graphs && !ctx->cfg.timing) {          // timing mode: per-kernel events, direct launches
    const std::vector<int64_t> key = {
        (int64_t)(uintptr_t)x, (int64_t)(uintptr_t)y, (int64_t)sizeof(E), P.g3[0], P.g3[1], P.g3[2],
        P.run_p1, P.run_deriv, P.run_ac, P.run_ssim, P.run_pdf, P.W, P.kind, P.T, P.nb,
        P.step[0], P.step[1], P.step[2], ctx->cfg.ssim_range_mode,
        (int64_t)(uintptr_t)ctx->cfg.debug_wssim, (int64_t)(uintptr_t)ctx->cfg.debug_der,
        (int64_t)(uintptr_t)ctx->parts, (int64_t)ctx->parts_cap};
    if (!ctx->gexec || key != ctx->gkey) {
      if (ctx->gexec) { cudaGraphExecDestroy(ctx->gexec); ctx->gexec = nullptr; }
      cudaGraph_t g = nullptr;
      if (cudaStreamBeginCapture(s, cudaStreamCaptureModeRelaxed) == cudaSuccess) {
        const czc_status cst = enqueue_single(ctx, P, x, y, F, sp);
        const cudaError_t ce = cudaStreamEndCapture(s, &g);
        if (cst == CZC_OK && ce == cudaSuccess && g &&
            cudaGraphInstantiate(&ctx->gexec, g, 0) == cudaSuccess)
          ctx->gkey = key;
        else
          ctx->gexec = nullptr;
        if (g) cudaGraphDestroy(g);
      }
      (void)cudaGetLastError();                          // a failed capture falls back to launches
    }
    if (ctx->gexec) {
      CZC_CUDA(ctx, cudaGraphLaunch(ctx->gexec, s));
      launched = true;
    }
  }
  if (!launched && (st = enqueue_single(ctx, P, x, y, F, sp)) != CZC_OK) return st;
  CZC_CUDA(ctx, cudaStreamSynchronize(s));
  combine_and_finish(P, ctx->hrec, 1, mask, out);
  finish_timing(ctx, out);
  return CZC_OK;
}

// Field view of one slab [z0, z0 + nzl) whose halo planes live in ctx->halo (lo: hlo planes,
// hi: hhi planes; filled by NCCL receives or, in loopback mode, device copies).
template <typename E>
static Field3<E> slab_field(czc_ctx* ctx, const Plan& P, const E* x, const E* y, int64_t z0, int64_t nzl,
                            int64_t hlo, int64_t hhi, E** xlo, E** ylo, E** xhi, E** yhi) {
  const int64_t plane = P.g3[1] * P.g3[2];
  *xlo = static_cast<E*>(ctx->halo);
  *ylo = *xlo + hlo * plane;
  *xhi = *ylo + hlo * plane;
  *yhi = *xhi + hhi * plane;
  Field3<E> F{};
  F.nz = P.g3[0]; F.ny = P.g3[1]; F.nx = P.g3[2];
  F.zown0 = z0; F.zown1 = z0 + nzl;
  int k = 0;
  if (hlo) { F.xs[k] = *xlo; F.ys[k] = *ylo; F.zs[k] = z0 - hlo; k++; }
  F.xs[k] = x; F.ys[k] = y; F.zs[k] = z0; k++;
  if (hhi) { F.xs[k] = *xhi; F.ys[k] = *yhi; F.zs[k] = z0 + nzl; k++; }
  F.nseg = k;
  F.zs[k] = z0 + nzl + hhi;
  return F;
}

// Slab table check shared by both slab paths: slabs tile dims[0] in order and every slab holds
// at least the halo depth its lower neighbour needs.
static bool slabs_ok(const std::vector<std::pair<int64_t, int64_t>>& tab, int64_t nz, int64_t H) {
  for (size_t r = 0; r < tab.size(); r++) {
    const bool contiguous = r == 0 ? tab[r].first == 0 : tab[r].first == tab[r - 1].first + tab[r - 1].second;
    if (!contiguous || tab[r].second < 1) return false;
    if (r + 1 < tab.size() && tab[r + 1].second < std::min(H, nz - tab[r + 1].first)) return false;
  }
  return tab.back().first + tab.back().second == nz;
}

// Loopback: the multi-GPU algorithm on one GPU.  Slab k owns planes [z0_k, z0_k + n_k); its
// halos are device-copied into ctx->halo (the buffers NCCL receives into); P1 states are merged
// in slab order on the device before P2; per-slab records are combined in slab order on the host.
template <typename E>
static czc_status assess_loopback(czc_ctx* ctx, const Plan& P, const E* x, const E* y, czc_result* out,
                                  uint64_t mask) {
  const cudaStream_t s = ctx->stream;
  const bool timing = ctx->cfg.timing != 0;
  const int K = ctx->cfg.loopback_slabs;
  const int64_t nz = P.g3[0], plane = P.g3[1] * P.g3[2];
  if (P.D != 3 || nz < K) { ctx->last_error = "loopback slab mode needs a 3-D field with dims[0] >= slabs"; return CZC_ERR_SHAPE; }
  std::vector<std::pair<int64_t, int64_t>> tab(K);
  for (int k = 0; k < K; k++) {
    const int64_t a = nz * k / K, b = nz * (k + 1) / K;
    tab[k] = {a, b - a};
  }
  const int64_t H = halo_depth(P);
  if (!slabs_ok(tab, nz, H)) { ctx->last_error = "slabs thinner than the halo depth"; return CZC_ERR_SHAPE; }
  const SsimParams sp = ssim_params(P, ctx->cfg);
  Record* drec = (Record*)ctx->dgather;
  P1State* dst = (P1State*)ctx->dstates;
  // one halo allocation for all slabs (a reallocation between slabs would synchronise the device)
  czc_status st0 = ensure_buf(ctx, &ctx->halo, &ctx->halo_cap, 2 * (size_t)(1 + H) * plane * sizeof(E) + 16);
  if (st0 != CZC_OK) return st0;
  CZC_CUDA(ctx, cudaMemsetAsync(drec, 0, (size_t)K * sizeof(Record), s));
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[0], s));
  if (P.run_p1) {
    for (int k = 0; k < K; k++) {
      czc_status st = p1_local(ctx, P, x + tab[k].first * plane, y + tab[k].first * plane, tab[k].second * plane);
      if (st != CZC_OK) return st;
      CZC_CUDA(ctx, cudaMemcpyAsync(dst + k, &ctx->dres->rec.p1, sizeof(P1State), cudaMemcpyDeviceToDevice, s));
      CZC_CUDA(ctx, cudaMemcpyAsync(&drec[k].p1, &ctx->dres->rec.p1, sizeof(P1State), cudaMemcpyDeviceToDevice, s));
    }
    CZC_CUDA(ctx, launch_p1_combine(dst, K, ctx->dres, s));
  }
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[1], s));
  for (int k = 0; k < K; k++) {
    const int64_t z0 = tab[k].first, nzl = tab[k].second;
    const int64_t hlo = (P.run_deriv && z0 > 0) ? 1 : 0;
    const int64_t hhi = std::min(H, nz - (z0 + nzl));
    czc_status st;
    E *xlo, *ylo, *xhi, *yhi;
    const Field3<E> F = slab_field(ctx, P, x + z0 * plane, y + z0 * plane, z0, nzl, hlo, hhi, &xlo, &ylo, &xhi, &yhi);
    const size_t pb = (size_t)plane * sizeof(E);
    if (hlo) {
      CZC_CUDA(ctx, cudaMemcpyAsync(xlo, x + (z0 - 1) * plane, pb, cudaMemcpyDeviceToDevice, s));
      CZC_CUDA(ctx, cudaMemcpyAsync(ylo, y + (z0 - 1) * plane, pb, cudaMemcpyDeviceToDevice, s));
    }
    if (hhi) {
      CZC_CUDA(ctx, cudaMemcpyAsync(xhi, x + (z0 + nzl) * plane, hhi * pb, cudaMemcpyDeviceToDevice, s));
      CZC_CUDA(ctx, cudaMemcpyAsync(yhi, y + (z0 + nzl) * plane, hhi * pb, cudaMemcpyDeviceToDevice, s));
    }
    if (P.run_pdf)
      CZC_CUDA(ctx, launch_pdf(x + z0 * plane, y + z0 * plane, nzl * plane, P.nb, ctx->p1_grid_cap, ctx->dres, s));
    if ((st = run_p23(ctx, P, F, sp)) != CZC_OK) return st;
    CZC_CUDA(ctx, cudaMemcpyAsync(drec[k].deriv, ctx->dres->rec.deriv,
                                  sizeof(Record) - offsetof(Record, deriv), cudaMemcpyDeviceToDevice, s));
  }
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[4], s));
  CZC_CUDA(ctx, copy_records(ctx->hrec, drec, K, P.run_pdf, s));
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[5], s));
  CZC_CUDA(ctx, cudaStreamSynchronize(s));
  combine_and_finish(P, ctx->hrec, K, mask, out);
  finish_timing(ctx, out);
  return CZC_OK;
}

// NCCL slab mode: this rank holds planes [z0, z0 + nzl) of the global field.
//  * Slab table: when this rank's call signature (its slab, the global shape, the halo depth, the
//    element type) differs from the last call's, every buffer the signature needs is allocated
//    FIRST and the slab table is all-gathered together with each rank's allocation status, so a
//    local failure is a collective decision (no rank leaves a peer waiting in a
//    collective) and a bad decomposition fails on every rank.  A repeated signature skips that
//    allgather and its host synchronisation; a 16-byte allgather at the end of the call still
//    checks that every rank kept its slab (a changed decomposition returns CZC_ERR_SHAPE on all
//    ranks and is re-validated on the next call).
//  * Halo exchange: grouped send / recv on the halo communicator and stream, ordered after the
//    caller's inputs, overlapping P1 and the P1-state allgather on the compute stream; P2 / P3
//    wait for it (an event).
//  * Collectives on the compute stream: the P1 states (merged in rank order on the device: every
//    rank needs the global mu_e, sigma_e^2), then the per-rank records (combined in rank order on
//    the host by combine_and_finish, the code exported as czc_combine).
//  * A CUDA / NCCL failure after the first collective of a call aborts this rank's communicators
//    (its queued operations are dropped) and the context returns CZC_ERR_COMM from then on.
template <typename E>
static czc_status assess_ranks(czc_ctx* ctx, const Plan& P, const E* x, const E* y, const czc_shape* shape,
                               czc_result* out, uint64_t mask) {
  const cudaStream_t s = ctx->stream, hs = ctx->halo_stream;
  const bool timing = ctx->cfg.timing != 0;
  if (!comm_usable(ctx->comm)) { ctx->last_error = "communicator aborted by an earlier failure"; return CZC_ERR_COMM; }
  const int nranks = comm_size(ctx->comm), rank = comm_rank(ctx->comm);
  const int64_t nz = P.g3[0], plane = P.g3[1] * P.g3[2];
  if (P.D != 3 || shape->dims[0] != nz) { ctx->last_error = "slab mode needs a 3-D field split along dims[0]"; return CZC_ERR_SHAPE; }
  const int64_t z0 = shape->z0, nzl = shape->nz_local > 0 ? shape->nz_local : nz;
  const int64_t H = halo_depth(P);
  // halo: H planes up from rank+1, one plane (derivatives) down from rank-1
  const int64_t hlo = (P.run_deriv && z0 > 0) ? 1 : 0;
  const int64_t hhi = std::min(H, nz - (z0 + nzl));
  const int64_t prev_hhi = rank > 0 ? std::min(H, nz - z0) : 0;
  const bool next_lo = P.run_deriv && rank + 1 < nranks;
  const size_t pb = (size_t)plane * sizeof(E);
  const SsimParams sp = ssim_params(P, ctx->cfg);
  E *xlo, *ylo, *xhi, *yhi;
  // the call signature: everything the buffers and the scratch layout depend on
  const std::vector<int64_t> key = {z0, nzl, nz, P.g3[1], P.g3[2], H, (int64_t)sizeof(E), P.run_p1, P.run_deriv,
                                    P.run_ac, P.run_ssim, P.run_pdf, P.W, P.T, P.kind, P.step[0], P.step[1], P.step[2]};
  if (key != ctx->slab_key) {
    ctx->slab_key.clear();
    // allocate first (halo planes, kernel scratch), then one collective decision
    czc_status local = ensure_buf(ctx, &ctx->halo, &ctx->halo_cap, 2 * (size_t)(hlo + hhi) * pb + 16);
    if (local == CZC_OK) {
      const Field3<E> F0 = slab_field(ctx, P, x, y, z0, nzl, hlo, hhi, &xlo, &ylo, &xhi, &yhi);
      local = ensure_scratch(ctx, P, F0, sp);
    }
    if (local == CZC_OK) local = ensure_buf(ctx, &ctx->parts, &ctx->parts_cap, (size_t)ctx->p1_grid_cap * sizeof(P1State));
    int64_t* pin = ctx->hpin;
    pin[0] = z0;
    pin[1] = nzl;
    pin[2] = (int64_t)local;
    CZC_CUDA(ctx, cudaMemcpyAsync(ctx->dgather_in, pin, 3 * sizeof(int64_t), cudaMemcpyHostToDevice, s));
    if (!comm_allgather(ctx->comm, ctx->dgather_in, ctx->dgather, 3 * sizeof(int64_t), s, &ctx->last_error)) return CZC_ERR_COMM;
    CZC_CUDA(ctx, cudaMemcpyAsync(pin + 3, ctx->dgather, 3 * (size_t)nranks * sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CZC_CUDA(ctx, cudaStreamSynchronize(s));
    const std::vector<int64_t> flat(pin + 3, pin + 3 + 3 * nranks);
    for (int r = 0; r < nranks; r++)
      if (flat[3 * r + 2] != CZC_OK) {
        ctx->last_error = "rank " + std::to_string(r) + " could not set up its slab: " + czc_strerror((czc_status)flat[3 * r + 2]);
        return (czc_status)flat[3 * r + 2];
      }
    std::vector<std::pair<int64_t, int64_t>> tab(nranks);
    for (int r = 0; r < nranks; r++) tab[r] = {flat[3 * r], flat[3 * r + 1]};
    if (!slabs_ok(tab, nz, H)) { ctx->last_error = "slabs must tile dims[0] in rank order, each >= the halo depth"; return CZC_ERR_SHAPE; }
    ctx->slab_tab.assign(2 * nranks, 0);
    for (int r = 0; r < nranks; r++) { ctx->slab_tab[2 * r] = tab[r].first; ctx->slab_tab[2 * r + 1] = tab[r].second; }
    ctx->slab_key = key;
  }
  // from here on every buffer exists; a failure aborts the communicators (see above)
  auto fail = [&](czc_status st) {
    comm_abort(ctx->comm);
    ctx->slab_key.clear();
    return st;
  };
#define CZC_SLAB(call)                                                              \
  do {                                                                              \
    cudaError_t _e = (call);                                                        \
    if (_e != cudaSuccess) return fail(cuda_fail(ctx, _e, #call));                  \
  } while (0)
  const Field3<E> F = slab_field(ctx, P, x, y, z0, nzl, hlo, hhi, &xlo, &ylo, &xhi, &yhi);
  if (timing) CZC_SLAB(cudaEventRecord(ctx->ev[0], s));
  // halo exchange on the halo stream, after the caller's writes of x / y (and this context's
  // previous kernels, which read the halo buffers) on the compute stream
  CZC_SLAB(cudaEventRecord(ctx->halo_ev[0], s));
  CZC_SLAB(cudaStreamWaitEvent(hs, ctx->halo_ev[0], 0));
  if (!comm_group_begin(&ctx->last_error)) return fail(CZC_ERR_COMM);
  bool ok = true;
  if (rank > 0 && prev_hhi > 0) {
    ok &= comm_send(ctx->comm, x, prev_hhi * pb, rank - 1, hs, &ctx->last_error);
    ok &= comm_send(ctx->comm, y, prev_hhi * pb, rank - 1, hs, &ctx->last_error);
  }
  if (next_lo) {
    ok &= comm_send(ctx->comm, x + (nzl - 1) * plane, pb, rank + 1, hs, &ctx->last_error);
    ok &= comm_send(ctx->comm, y + (nzl - 1) * plane, pb, rank + 1, hs, &ctx->last_error);
  }
  if (hhi > 0) {
    ok &= comm_recv(ctx->comm, xhi, hhi * pb, rank + 1, hs, &ctx->last_error);
    ok &= comm_recv(ctx->comm, yhi, hhi * pb, rank + 1, hs, &ctx->last_error);
  }
  if (hlo > 0) {
    ok &= comm_recv(ctx->comm, xlo, pb, rank - 1, hs, &ctx->last_error);
    ok &= comm_recv(ctx->comm, ylo, pb, rank - 1, hs, &ctx->last_error);
  }
  if (!comm_group_end(&ctx->last_error) || !ok) return fail(CZC_ERR_COMM);
  CZC_SLAB(cudaEventRecord(ctx->halo_ev[1], hs));
  // The derivatives and local-range SSIM need only the slab and its halo: without per-kernel
  // timing they run on the second stream as soon as the halo is in (the single-GPU branch
  // layout, enqueue_single), concurrently with P1, its allgather and AC on the compute stream.
  const bool branch = !timing && ctx->concurrent;
  const bool ssim_early = P.run_ssim && sp.range_mode == 0;
  czc_status st = CZC_OK;
  if (branch) {
    CZC_SLAB(cudaStreamWaitEvent(ctx->stream2, ctx->halo_ev[1], 0));
    if (P.run_deriv && (st = launch_deriv_k(ctx, F, ctx->stream2)) != CZC_OK) return fail(st);
    if (ssim_early && (st = launch_ssim_k(ctx, P, F, sp, ctx->stream2)) != CZC_OK) return fail(st);
  }
  // P1 on the local slab (overlaps the halo transfer), one small allgather of the states, merged
  // in rank order on the device
  if (P.run_p1) {
    CZC_SLAB(launch_p1(x, y, nzl * plane, ctx->p1_grid_cap, (P1State*)ctx->parts, ctx->dres, ctx->tickets + TICKET_P1, s));
    if (!comm_allgather(ctx->comm, &ctx->dres->rec.p1, ctx->dstates, sizeof(P1State), s, &ctx->last_error)) return fail(CZC_ERR_COMM);
    CZC_SLAB(launch_p1_combine((const P1State*)ctx->dstates, nranks, ctx->dres, s));
  }
  if (P.run_pdf) CZC_SLAB(launch_pdf(x, y, nzl * plane, P.nb, ctx->p1_grid_cap, ctx->dres, s));
  if (timing) CZC_SLAB(cudaEventRecord(ctx->ev[1], s));
  CZC_SLAB(cudaStreamWaitEvent(s, ctx->halo_ev[1], 0));
  if (branch) {                                          // scratch sized above: no allocation
    if (P.run_ac && (st = launch_ac_k(ctx, P, F, s)) != CZC_OK) return fail(st);
    if (P.run_ssim && !ssim_early && (st = launch_ssim_k(ctx, P, F, sp, s)) != CZC_OK) return fail(st);
    CZC_SLAB(cudaEventRecord(ctx->join_ev, ctx->stream2));
    CZC_SLAB(cudaStreamWaitEvent(s, ctx->join_ev, 0));
  } else if ((st = run_p23(ctx, P, F, sp)) != CZC_OK) {
    return fail(st);
  }
  if (timing) CZC_SLAB(cudaEventRecord(ctx->ev[4], s));
  // every rank's record, combined in rank order on the host; plus the slab check of this call
  if (!comm_allgather(ctx->comm, &ctx->dres->rec, ctx->dgather, sizeof(Record), s, &ctx->last_error)) return fail(CZC_ERR_COMM);
  CZC_SLAB(copy_records(ctx->hrec, (const Record*)ctx->dgather, nranks, P.run_pdf, s));
  // (pinned staging: a pageable copy would block the host until the kernels above finish)
  int64_t* pin = ctx->hpin;            // [0, 2): this rank's slab, [2, 2 + 2 nranks): the gathered table
  pin[0] = z0;
  pin[1] = nzl;
  CZC_SLAB(cudaMemcpyAsync(ctx->dgather_in, pin, 2 * sizeof(int64_t), cudaMemcpyHostToDevice, s));
  if (!comm_allgather(ctx->comm, ctx->dgather_in, ctx->dstates, 2 * sizeof(int64_t), s, &ctx->last_error)) return fail(CZC_ERR_COMM);
  CZC_SLAB(cudaMemcpyAsync(pin + 2, ctx->dstates, 2 * (size_t)nranks * sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  if (timing) CZC_SLAB(cudaEventRecord(ctx->ev[5], s));
  CZC_SLAB(cudaStreamSynchronize(s));
#undef CZC_SLAB
  const std::vector<int64_t> now(pin + 2, pin + 2 + 2 * nranks);
  if (now != ctx->slab_tab) {          // some rank changed its slab without the others
    ctx->slab_key.clear();
    ctx->last_error = "the slab decomposition changed on some ranks but not on others";
    return CZC_ERR_SHAPE;
  }
  combine_and_finish(P, ctx->hrec, nranks, mask, out);
  finish_timing(ctx, out);
  return CZC_OK;
}

static czc_status check_common(czc_ctx* ctx, const void* orig, const void* recon, const czc_shape* shape,
                               czc_dtype dtype, czc_result* out) {
  if (!out) return CZC_ERR_INVALID;
  memset(out, 0, sizeof(*out));
  if (!ctx || !orig || !recon || !shape) return CZC_ERR_INVALID;
  if (dtype != CZC_F32 && dtype != CZC_F64) {
    ctx->last_error = "dtype must be CZC_F32 or CZC_F64";
    return CZC_ERR_DTYPE;
  }
  return CZC_OK;
}

// Four active axes (NEXT row f3): P1 / PDF on the flat pair, then the generic 4-D stencil,
// autocorrelation and window kernels (p4_generic.cu); single GPU only.
template <typename E>
static czc_status assess_4d(czc_ctx* ctx, const Plan& P, const E* x, const E* y, czc_result* out, uint64_t mask) {
  const cudaStream_t s = ctx->stream;
  const bool timing = ctx->cfg.timing != 0;
  const int64_t N = P.g4[0] * P.g4[1] * P.g4[2] * P.g4[3];
  const size_t need = std::max((size_t)ctx->p1_grid_cap * sizeof(P1State),
                               (size_t)g4_max_blocks(ctx->sm_count) * kAcSlots * sizeof(double));
  czc_status st = ensure_buf(ctx, &ctx->parts, &ctx->parts_cap, need);
  if (st != CZC_OK) return st;
  double* parts = (double*)ctx->parts;
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[0], s));
  if ((st = p1_local(ctx, P, x, y, N)) != CZC_OK) return st;
  if (P.run_pdf) CZC_CUDA(ctx, launch_pdf(x, y, N, P.nb, ctx->p1_grid_cap, ctx->dres, s));
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[1], s));
  if (P.run_deriv)
    CZC_CUDA(ctx, launch_deriv4(x, y, P.g4, ctx->sm_count, parts, ctx->dres, ctx->tickets + TICKET_DERIV, ctx->cfg.debug_der, s));
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[2], s));
  if (P.run_ac) CZC_CUDA(ctx, launch_ac4(x, y, P.g4, P.T, ctx->sm_count, parts, ctx->dres, ctx->tickets + TICKET_ACZ, s));
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[3], s));
  if (P.run_ssim)
    CZC_CUDA(ctx, launch_ssim4(x, y, P.g4, P.win4, P.step4, ctx->cfg.ssim_range_mode, ctx->sm_count, parts, ctx->dres,
                               ctx->tickets + TICKET_SSIM, ctx->cfg.debug_wssim, s));
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[4], s));
  CZC_CUDA(ctx, copy_records(ctx->hrec, &ctx->dres->rec, 1, P.run_pdf, s));
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[5], s));
  CZC_CUDA(ctx, cudaStreamSynchronize(s));
  combine_and_finish(P, ctx->hrec, 1, mask, out);
  finish_timing(ctx, out);
  return CZC_OK;
}

template <typename E>
static czc_status assess_dispatch(czc_ctx* ctx, const Plan& P, const E* x, const E* y, const czc_shape* shape,
                                  czc_result* out, uint64_t mask) {
  if (P.D == 4) {
    if (ctx->comm || ctx->cfg.loopback_slabs > 1) {
      ctx->last_error = "4-D fields run on one GPU (no slab mode)";
      return CZC_ERR_UNSUPPORTED;
    }
    return assess_4d(ctx, P, x, y, out, mask);
  }
  if (ctx->comm) return assess_ranks(ctx, P, x, y, shape, out, mask);
  if (ctx->cfg.loopback_slabs > 1) return assess_loopback(ctx, P, x, y, out, mask);
  return assess_single(ctx, P, x, y, out, mask);
}

// The fields must be memory the context's device can read: device memory of that device (or
// managed / mapped host memory).  Unregistered host memory or another device's allocation would
// fault inside a kernel and leave a sticky error in the CUDA context, so it is a
// status code here instead.
static czc_status check_device_ptr(czc_ctx* ctx, const void* p, const char* what) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    (void)cudaGetLastError();
    ctx->last_error = std::string(what) + ": not a CUDA-accessible pointer";
    return CZC_ERR_INVALID;
  }
  if (a.type == cudaMemoryTypeUnregistered) {
    ctx->last_error = std::string(what) + ": host memory (czc_assess takes device pointers; see czc_assess_host)";
    return CZC_ERR_INVALID;
  }
  if (a.type == cudaMemoryTypeDevice && a.device != ctx->device) {
    ctx->last_error = std::string(what) + ": memory of device " + std::to_string(a.device) +
                      ", context bound to device " + std::to_string(ctx->device);
    return CZC_ERR_INVALID;
  }
  return CZC_OK;
}

extern "C" czc_status czc_assess(czc_ctx* ctx, const void* orig, const void* recon, const czc_shape* shape,
                                 czc_dtype dtype, uint64_t metric_mask, czc_result* out) {
  czc_status st = check_common(ctx, orig, recon, shape, dtype, out);
  if (st != CZC_OK) return st;
  NvtxRange r_("czc/assess");
  if (cudaSetDevice(ctx->device) != cudaSuccess) return cuda_fail(ctx, cudaGetLastError(), "cudaSetDevice");
  if ((st = check_device_ptr(ctx, orig, "orig")) != CZC_OK || (st = check_device_ptr(ctx, recon, "recon")) != CZC_OK)
    return st;
  Plan P;
  st = make_plan(ctx->cfg, shape->ndim, shape->dims, metric_mask, P, ctx->last_error);
  if (st == CZC_OK) {
    const int64_t nzl = shape->nz_local > 0 ? shape->nz_local : shape->dims[0];
    if (shape->z0 < 0 || shape->z0 + nzl > shape->dims[0]) {
      ctx->last_error = "slab [z0, z0+nz_local) outside dims[0]";
      st = CZC_ERR_SHAPE;
    } else if (!ctx->comm && (shape->z0 != 0 || nzl != shape->dims[0])) {
      ctx->last_error = "a slab shape needs nranks > 1";
      st = CZC_ERR_SHAPE;
    } else if (dtype == CZC_F64) {
      st = assess_dispatch(ctx, P, (const double*)orig, (const double*)recon, shape, out, metric_mask);
    } else {
      st = assess_dispatch(ctx, P, (const float*)orig, (const float*)recon, shape, out, metric_mask);
    }
  }
  if (st != CZC_OK) out->computed_mask = 0;
  return st;
}

// Pipelined host path (single GPU, 3-D field): the pair is copied host->device in K z-chunks on a
// copy stream while P1, the derivatives and SSIM of chunk k run on the compute stream as soon as
// chunk k and the halo planes above it have arrived (records per chunk, owned ranges as in slab
// mode); the autocorrelation, which needs the global mean / variance of the error, runs once the
// whole field is resident.  Same combine as slab mode.
template <typename E>
static czc_status assess_host_pipelined(czc_ctx* ctx, const Plan& P, const E* hx, const E* hy,
                                        czc_result* out, uint64_t mask, int K) {
  const cudaStream_t s = ctx->stream;
  const bool timing = ctx->cfg.timing != 0;
  const int64_t nz = P.g3[0], plane = P.g3[1] * P.g3[2];
  const size_t pb = (size_t)plane * sizeof(E);
  E* x = static_cast<E*>(ctx->din[0]);
  E* y = static_cast<E*>(ctx->din[1]);
  if (!ctx->copy_stream[0]) {
    for (int c = 0; c < 2; c++) {
      CZC_CUDA(ctx, cudaStreamCreateWithFlags(&ctx->copy_stream[c], cudaStreamNonBlocking));
      for (int i = 0; i < kMaxHostChunks; i++)
        CZC_CUDA(ctx, cudaEventCreateWithFlags(&ctx->copy_ev[c][i], cudaEventDisableTiming));
    }
  }
  std::vector<int64_t> b(K + 1);
  for (int k = 0; k <= K; k++) b[k] = nz * k / K;
  // the copy streams start after everything already queued on the compute stream (which may
  // still read the device buffers of the previous call)
  CZC_CUDA(ctx, cudaEventRecord(ctx->copy_ev[0][0], s));
  CZC_CUDA(ctx, cudaStreamWaitEvent(ctx->copy_stream[0], ctx->copy_ev[0][0], 0));
  for (int k = 0; k < K; k++) {
    const size_t bytes = (size_t)(b[k + 1] - b[k]) * pb;
    CZC_CUDA(ctx, cudaMemcpyAsync(x + b[k] * plane, hx + b[k] * plane, bytes, cudaMemcpyHostToDevice, ctx->copy_stream[0]));
    CZC_CUDA(ctx, cudaMemcpyAsync(y + b[k] * plane, hy + b[k] * plane, bytes, cudaMemcpyHostToDevice, ctx->copy_stream[0]));
    CZC_CUDA(ctx, cudaEventRecord(ctx->copy_ev[0][k], ctx->copy_stream[0]));
  }
  Field3<E> F{};
  F.nz = nz; F.ny = P.g3[1]; F.nx = P.g3[2];
  F.nseg = 1; F.xs[0] = x; F.ys[0] = y; F.zs[0] = 0; F.zs[1] = nz;
  const SsimParams sp = ssim_params(P, ctx->cfg);
  Record* drec = (Record*)ctx->dgather;
  P1State* dst = (P1State*)ctx->dstates;
  CZC_CUDA(ctx, cudaMemsetAsync(drec, 0, (size_t)K * sizeof(Record), s));
  // Per arrived chunk k (planes < b[k+1] resident): P1 of the chunk, then the derivative points
  // and SSIM window origins whose whole stencil / window is resident — owned ranges
  // [done, b[k+1] - 1) and [done, b[k+1] - W + 1) (the whole rest for the last chunk), so no
  // chunk waits for the next one and only the last chunk's share runs after the last copy.
  Plan Pd = P, Ps = P;
  Pd.run_ac = Pd.run_ssim = false;
  Ps.run_ac = Ps.run_deriv = false;
  int64_t d_done = 0, s_done = 0;
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[0], s));
  for (int k = 0; k < K; k++) {
    CZC_CUDA(ctx, cudaStreamWaitEvent(s, ctx->copy_ev[0][k], 0));
    const bool last = k == K - 1;
    if (P.run_p1) {
      czc_status st = p1_local(ctx, P, x + b[k] * plane, y + b[k] * plane, (b[k + 1] - b[k]) * plane);
      if (st != CZC_OK) return st;
      CZC_CUDA(ctx, cudaMemcpyAsync(dst + k, &ctx->dres->rec.p1, sizeof(P1State), cudaMemcpyDeviceToDevice, s));
      CZC_CUDA(ctx, cudaMemcpyAsync(&drec[k].p1, &ctx->dres->rec.p1, sizeof(P1State), cudaMemcpyDeviceToDevice, s));
    }
    if (P.run_deriv) {                                 // possibly empty: the record then holds identities
      const int64_t hi = std::max(d_done, last ? nz : b[k + 1] - 1);
      F.zown0 = d_done;
      F.zown1 = hi;
      czc_status st = run_p23(ctx, Pd, F, sp);
      if (st != CZC_OK) return st;
      CZC_CUDA(ctx, cudaMemcpyAsync(drec[k].deriv, ctx->dres->rec.deriv, sizeof(drec[k].deriv), cudaMemcpyDeviceToDevice, s));
      d_done = hi;
    }
    if (P.run_ssim) {
      const int64_t hi = std::max(s_done, last ? nz : b[k + 1] - (P.W - 1));
      F.zown0 = s_done;
      F.zown1 = hi;
      czc_status st = run_p23(ctx, Ps, F, sp);
      if (st != CZC_OK) return st;
      CZC_CUDA(ctx, cudaMemcpyAsync(drec[k].ssim, ctx->dres->rec.ssim, sizeof(drec[k].ssim), cudaMemcpyDeviceToDevice, s));
      s_done = hi;
    }
  }
  if (P.run_p1) CZC_CUDA(ctx, launch_p1_combine(dst, K, ctx->dres, s));
  if (P.run_pdf) {
    CZC_CUDA(ctx, launch_pdf(x, y, nz * plane, P.nb, ctx->p1_grid_cap, ctx->dres, s));
    CZC_CUDA(ctx, cudaMemcpyAsync(drec[0].pdf, ctx->dres->rec.pdf, sizeof(drec[0].pdf), cudaMemcpyDeviceToDevice, s));
  }
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[1], s));
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[2], s));
  if (P.run_ac) {
    F.zown0 = 0;
    F.zown1 = nz;
    czc_status st = ensure_scratch(ctx, P, F, sp);
    if (st != CZC_OK) return st;
    CZC_CUDA(ctx, launch_ac(F, P.T, 0, parts_at(ctx, ctx->off_ac), ctx->dres, ctx->tickets + TICKET_ACZ, s));
    CZC_CUDA(ctx, cudaMemcpyAsync(drec[0].ac, ctx->dres->rec.ac, sizeof(drec[0].ac), cudaMemcpyDeviceToDevice, s));
  }
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[3], s));
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[4], s));
  CZC_CUDA(ctx, copy_records(ctx->hrec, drec, K, P.run_pdf, s));
  if (timing) CZC_CUDA(ctx, cudaEventRecord(ctx->ev[5], s));
  CZC_CUDA(ctx, cudaStreamSynchronize(s));
  combine_and_finish(P, ctx->hrec, K, mask, out);
  finish_timing(ctx, out);
  return CZC_OK;
}

extern "C" czc_status czc_assess_host(czc_ctx* ctx, const void* orig, const void* recon, const czc_shape* shape,
                                      czc_dtype dtype, uint64_t metric_mask, czc_result* out) {
  czc_status st = check_common(ctx, orig, recon, shape, dtype, out);
  if (st != CZC_OK) return st;
  NvtxRange r_("czc/assess_host");
  if (shape->ndim < 1 || shape->ndim > CZC_MAX_DIMS) return CZC_ERR_SHAPE;
  int64_t n = 1;
  for (int i = 0; i < shape->ndim; i++) {
    if (shape->dims[i] < 1) return CZC_ERR_SHAPE;
    n *= (i == 0 && shape->nz_local > 0) ? shape->nz_local : shape->dims[i];
  }
  if (cudaSetDevice(ctx->device) != cudaSuccess) return cuda_fail(ctx, cudaGetLastError(), "cudaSetDevice");
  const size_t bytes = (size_t)n * (dtype == CZC_F64 ? sizeof(double) : sizeof(float));
  if (bytes > ctx->din_cap) {
    cudaFree(ctx->din[0]);
    cudaFree(ctx->din[1]);
    ctx->din[0] = ctx->din[1] = nullptr;
    ctx->din_cap = 0;
    CZC_CUDA(ctx, cudaMalloc(&ctx->din[0], bytes));
    CZC_CUDA(ctx, cudaMalloc(&ctx->din[1], bytes));
    ctx->din_cap = bytes;
  }
  // pipelined path: single GPU, 3-D field, chunks at least as thick as the halo depth
  Plan P;
  std::string why;
  const bool plain = !ctx->comm && ctx->cfg.loopback_slabs <= 1 &&
                     make_plan(ctx->cfg, shape->ndim, shape->dims, metric_mask, P, why) == CZC_OK && P.D == 3 &&
                     (shape->nz_local == 0 || shape->nz_local == shape->dims[0]);
  if (plain) {
    // chunks of >= 4 planes, at most kHostChunks (CZC_HOST_CHUNKS overrides: A/B timing only)
    int kc = kHostChunks;
    if (const char* e = getenv("CZC_HOST_CHUNKS")) kc = std::max(2, std::min(kMaxHostChunks, atoi(e)));
    const int K = (int)std::min<int64_t>(kc, P.g3[0] / 4);
    if (K >= 2) {
      st = dtype == CZC_F64
               ? assess_host_pipelined(ctx, P, (const double*)orig, (const double*)recon, out, metric_mask, K)
               : assess_host_pipelined(ctx, P, (const float*)orig, (const float*)recon, out, metric_mask, K);
      if (st != CZC_OK) out->computed_mask = 0;
      return st;
    }
  }
  CZC_CUDA(ctx, cudaMemcpyAsync(ctx->din[0], orig, bytes, cudaMemcpyHostToDevice, ctx->stream));
  CZC_CUDA(ctx, cudaMemcpyAsync(ctx->din[1], recon, bytes, cudaMemcpyHostToDevice, ctx->stream));
  return czc_assess(ctx, ctx->din[0], ctx->din[1], shape, dtype, metric_mask, out);
}

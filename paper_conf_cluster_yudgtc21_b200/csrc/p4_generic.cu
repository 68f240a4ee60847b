// p4_generic.cu — the stencil, autocorrelation and SSIM patterns for 4-D fields (NEXT row f3).
//
// Paper: L92 — the kernels "can be easily extended to other dimensions (including 1D, 2D, and
// 4D)"; the paper evaluates 3-D data only (L330).  The definitions are those of the 3-D engines
// with a fourth axis (R9-R17 over the active axes, D = 4):
//   Der1 = sum_a |f(p+e_a) - f(p-e_a)| (Eq. 1), Der2 / Lap / Div / Grad as in R9 (L129,
//   Alg. 2), interior points of all four axes (R11);
//   AC(tau) = sum_{p in R_tau} eps_p (1/4) sum_a eps_{p+tau e_a} / ne / sigma^2 (Eq. 2);
//   local SSIM of every w0 x w1 x w2 x w3 window (L139-L146), range L of the original window.
// These are generic grid-stride kernels (one point or one window per thread step, neighbours
// through L1/L2) rather than the streamed, register-ring designs of the 3-D engines: 4-D fields
// are a correctness extension here, not a tuned path.  FP64 accumulation, block partials and the
// deterministic last-block finish are shared with the 3-D engines.
#include "czc_internal.cuh"

namespace czc {

constexpr int kG4Threads = 256;

template <typename T>
struct Field4 {
  const T* x;
  const T* y;
  int64_t n[4];      // extents, slowest first (all > 1)
  int64_t st[4];     // element strides
};

__device__ __forceinline__ void decode4(int64_t i, const int64_t len[4], int64_t c[4]) {
  c[3] = i % len[3]; i /= len[3];
  c[2] = i % len[2]; i /= len[2];
  c[1] = i % len[1];
  c[0] = i / len[1];
}

struct Deriv4Op {
  __device__ int operator()(int k) const { return deriv_op(k); }
};
struct Sum4Op {
  __device__ int operator()(int) const { return OP_SUM; }
};

// One derived-field set (Der1, Der2, Grad, Div, Lap) of f at linear index c over four axes.
template <typename T>
__device__ __forceinline__ void fields4(const T* __restrict__ f, int64_t c, const int64_t st[4], double F[CZC_NDERIV]) {
  const double f0 = f[c];
  double der1 = 0, der2 = 0, d2 = 0, dsum = 0, lap = 0;
#pragma unroll
  for (int a = 0; a < 4; a++) {
    const double p = __ldg(f + c + st[a]), m = __ldg(f + c - st[a]);
    const double delta = p - m, l = p - 2.0 * f0 + m;
    der1 += fabs(delta);
    der2 += fabs(l);
    d2 = fma(delta, delta, d2);
    dsum += delta;
    lap += l;
  }
  F[CZC_DER1] = der1;
  F[CZC_DER2] = der2;
  F[CZC_GRAD] = 0.5 * sqrt(d2);     // sqrt(sum (delta/2)^2), the /2 folded exactly
  F[CZC_DIV] = 0.5 * dsum;
  F[CZC_LAP] = lap;
}

template <typename T>
__global__ void __launch_bounds__(kG4Threads)
deriv4_kernel(Field4<T> s, double* __restrict__ parts, DevResults* __restrict__ res, unsigned int* __restrict__ ticket,
              double* __restrict__ dbg) {
  double acc[kDerivSlots];
#pragma unroll
  for (int k = 0; k < kDerivSlots; k++) acc[k] = op_identity(deriv_op(k));
  const int64_t len[4] = {s.n[0] - 2, s.n[1] - 2, s.n[2] - 2, s.n[3] - 2};
  const int64_t nI = len[0] * len[1] * len[2] * len[3];
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nI; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t c4[4];
    decode4(i, len, c4);
    const int64_t c = (c4[0] + 1) * s.st[0] + (c4[1] + 1) * s.st[1] + (c4[2] + 1) * s.st[2] + c4[3] + 1;
    double Fx[CZC_NDERIV], Fy[CZC_NDERIV];
    fields4(s.x, c, s.st, Fx);
    fields4(s.y, c, s.st, Fy);
#pragma unroll
    for (int fi = 0; fi < CZC_NDERIV; fi++) {
      const double d = Fy[fi] - Fx[fi];
      if (dbg) dbg[fi * nI + i] = d;               // czc_config.debug_der: C order of the interior
      acc[fi * kDerivStats + 0] = fmax(acc[fi * kDerivStats + 0], fabs(d));
      acc[fi * kDerivStats + 1] += fabs(d);
      acc[fi * kDerivStats + 2] = fma(d, d, acc[fi * kDerivStats + 2]);
      acc[fi * kDerivStats + 3] = fmin(acc[fi * kDerivStats + 3], Fx[fi]);
      acc[fi * kDerivStats + 4] = fmax(acc[fi * kDerivStats + 4], Fx[fi]);
    }
  }
  block_reduce_slots<kDerivSlots>(acc, Deriv4Op{}, parts + (size_t)blockIdx.x * kDerivSlots);
  if (!last_block_arrive(ticket)) return;
  finish_slots<kDerivSlots>(parts, gridDim.x, Deriv4Op{}, res->rec.deriv);
  if (threadIdx.x == 0) *ticket = 0;
}

// Eq. 2 over four axes: point p owns eps_p eps_{p + t e_a} for every axis a and every lag
// t <= lim(p) = min_b (n_b - 1 - p_b) (p in R_t), so the lag bound is one number per point.
template <typename T, int TM>
__global__ void __launch_bounds__(kG4Threads)
ac4_kernel(Field4<T> s, int T_, double* __restrict__ parts, DevResults* __restrict__ res, unsigned int* __restrict__ ticket) {
  const double mu = res->p1g.me;
  double acc[TM];
#pragma unroll
  for (int t = 0; t < TM; t++) acc[t] = 0;
  const int64_t N = s.n[0] * s.n[1] * s.n[2] * s.n[3];
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < N; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t c4[4];
    decode4(i, s.n, c4);
    int64_t lim = T_;
#pragma unroll
    for (int b = 0; b < 4; b++) lim = min(lim, s.n[b] - 1 - c4[b]);
    if (lim <= 0) continue;
    const double ep = ((double)s.y[i] - (double)s.x[i]) - mu;
#pragma unroll
    for (int t = 1; t <= TM; t++) {
      if (t > lim) break;
      double nb = 0;
#pragma unroll
      for (int a = 0; a < 4; a++) {
        const int64_t q = i + t * s.st[a];
        nb += ((double)__ldg(s.y + q) - (double)__ldg(s.x + q)) - mu;
      }
      acc[t - 1] = fma(ep, nb, acc[t - 1]);
    }
  }
  double rec[kAcSlots];
#pragma unroll
  for (int t = 0; t < kAcSlots; t++) rec[t] = t < TM ? acc[t] : 0.0;
  block_reduce_slots<kAcSlots>(rec, Sum4Op{}, parts + (size_t)blockIdx.x * kAcSlots);
  if (!last_block_arrive(ticket)) return;
  finish_slots<kAcSlots>(parts, gridDim.x, Sum4Op{}, res->rec.ac[0]);
  if (threadIdx.x == 0) *ticket = 0;
}

struct Ssim4Params {
  int w[4], s[4];
  int64_t nw[4];     // window-grid extents
  int range_mode;
};

// Local SSIM of every window of the grid, one window per thread step, by the plain definition
// (L139, readings R14-R15): two passes over the window's w0 w1 w2 w3 samples — FP64 means about
// the window's own first sample, exact min / max of x, then centred second moments — and the
// textbook mix.  No running sums, so no rounding error outlives its window (the 3-D engines'
// certificate is not needed here).
template <typename T>
__global__ void __launch_bounds__(kG4Threads)
ssim4_kernel(Field4<T> s, Ssim4Params p, double* __restrict__ parts, DevResults* __restrict__ res,
             unsigned int* __restrict__ ticket, double* __restrict__ dbg) {
  const double Lglob = res->p1g.xmax - res->p1g.xmin;
  const double invM = 1.0 / (double)(p.w[0] * p.w[1] * p.w[2] * p.w[3]);
  const int64_t total = p.nw[0] * p.nw[1] * p.nw[2] * p.nw[3];
  double ssum = 0, scnt = 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t c4[4];
    decode4(i, p.nw, c4);
    const int64_t o = c4[0] * p.s[0] * s.st[0] + c4[1] * p.s[1] * s.st[1] + c4[2] * p.s[2] * s.st[2] + c4[3] * p.s[3];
    const double K = s.x[o];
    double sx = 0, sy = 0;
    T mn = s.x[o], mx = mn;
    for (int l = 0; l < p.w[0]; l++)
      for (int k = 0; k < p.w[1]; k++)
        for (int j = 0; j < p.w[2]; j++) {
          const int64_t r = o + l * s.st[0] + k * s.st[1] + j * s.st[2];
          for (int q = 0; q < p.w[3]; q++) {
            const T xv = __ldg(s.x + r + q), yv = __ldg(s.y + r + q);
            sx += (double)xv - K;
            sy += (double)yv - K;
            mn = tmin(mn, xv);
            mx = tmax(mx, xv);
          }
        }
    const double mux = K + sx * invM, muy = K + sy * invM;
    double vx = 0, vy = 0, cxy = 0;
    for (int l = 0; l < p.w[0]; l++)
      for (int k = 0; k < p.w[1]; k++)
        for (int j = 0; j < p.w[2]; j++) {
          const int64_t r = o + l * s.st[0] + k * s.st[1] + j * s.st[2];
          for (int q = 0; q < p.w[3]; q++) {
            const double dx = (double)__ldg(s.x + r + q) - mux, dy = (double)__ldg(s.y + r + q) - muy;
            vx = fma(dx, dx, vx);
            vy = fma(dy, dy, vy);
            cxy = fma(dx, dy, cxy);
          }
        }
    vx *= invM;
    vy *= invM;
    cxy *= invM;
    double L = p.range_mode ? Lglob : (double)mx - (double)mn;
    L = (L == 0.0) ? 1.0 : L;
    const double C1 = (0.01 * L) * (0.01 * L), C2 = (0.03 * L) * (0.03 * L);
    const double ssim = ((2.0 * mux * muy + C1) * (2.0 * cxy + C2)) / ((mux * mux + muy * muy + C1) * (vx + vy + C2));
    ssum += ssim;
    scnt += 1.0;
    if (dbg) dbg[i] = ssim;
  }
  double rec[kSsimSlots] = {ssum, scnt, 0.0};
  block_reduce_slots<kSsimSlots>(rec, Sum4Op{}, parts + (size_t)blockIdx.x * kSsimSlots);
  if (!last_block_arrive(ticket)) return;
  finish_slots<kSsimSlots>(parts, gridDim.x, Sum4Op{}, res->rec.ssim);
  if (threadIdx.x == 0) *ticket = 0;
}

template <typename T>
static Field4<T> field4(const T* x, const T* y, const int64_t n[4]) {
  Field4<T> f;
  f.x = x; f.y = y;
  for (int a = 0; a < 4; a++) f.n[a] = n[a];
  f.st[3] = 1;
  for (int a = 2; a >= 0; a--) f.st[a] = f.st[a + 1] * n[a + 1];
  return f;
}

static unsigned g4_grid(int64_t work, int sms) {
  int64_t b = (work + kG4Threads - 1) / kG4Threads;
  const int64_t cap = (int64_t)sms * 8;
  if (b > cap) b = cap;
  return (unsigned)(b < 1 ? 1 : b);
}

// Blocks of the largest 4-D launch (scratch sizing): every grid is capped at 8 blocks per SM.
int64_t g4_max_blocks(int sms) { return (int64_t)sms * 8; }

template <typename T>
cudaError_t launch_deriv4(const T* x, const T* y, const int64_t n[4], int sms, double* parts, DevResults* res,
                          unsigned int* ticket, double* dbg, cudaStream_t st) {
  const Field4<T> f = field4(x, y, n);
  const int64_t nI = (n[0] - 2) * (n[1] - 2) * (n[2] - 2) * (n[3] - 2);
  deriv4_kernel<T><<<g4_grid(nI, sms), kG4Threads, 0, st>>>(f, parts, res, ticket, dbg);
  return cudaGetLastError();
}

template <typename T>
cudaError_t launch_ac4(const T* x, const T* y, const int64_t n[4], int T_, int sms, double* parts, DevResults* res,
                       unsigned int* ticket, cudaStream_t st) {
  const Field4<T> f = field4(x, y, n);
  cudaError_t e = cudaMemsetAsync(res->rec.ac, 0, sizeof(res->rec.ac), st);
  if (e != cudaSuccess) return e;
  const unsigned g = g4_grid(n[0] * n[1] * n[2] * n[3], sms);
  if (T_ <= 4) ac4_kernel<T, 4><<<g, kG4Threads, 0, st>>>(f, T_, parts, res, ticket);
  else if (T_ <= 10) ac4_kernel<T, 10><<<g, kG4Threads, 0, st>>>(f, T_, parts, res, ticket);
  else ac4_kernel<T, 16><<<g, kG4Threads, 0, st>>>(f, T_, parts, res, ticket);
  return cudaGetLastError();
}

template <typename T>
cudaError_t launch_ssim4(const T* x, const T* y, const int64_t n[4], const int w[4], const int stp[4], int range_mode,
                         int sms, double* parts, DevResults* res, unsigned int* ticket, double* dbg, cudaStream_t st) {
  const Field4<T> f = field4(x, y, n);
  Ssim4Params p;
  int64_t total = 1;
  for (int a = 0; a < 4; a++) {
    p.w[a] = w[a];
    p.s[a] = stp[a];
    p.nw[a] = (n[a] - w[a]) / stp[a] + 1;
    total *= p.nw[a];
  }
  p.range_mode = range_mode;
  ssim4_kernel<T><<<g4_grid(total, sms), kG4Threads, 0, st>>>(f, p, parts, res, ticket, dbg);
  return cudaGetLastError();
}

#define CZC_G4_INST(T)                                                                                         \
  template cudaError_t launch_deriv4<T>(const T*, const T*, const int64_t*, int, double*, DevResults*,         \
                                        unsigned int*, double*, cudaStream_t);                                 \
  template cudaError_t launch_ac4<T>(const T*, const T*, const int64_t*, int, int, double*, DevResults*,       \
                                     unsigned int*, cudaStream_t);                                             \
  template cudaError_t launch_ssim4<T>(const T*, const T*, const int64_t*, const int*, const int*, int, int,   \
                                       double*, DevResults*, unsigned int*, double*, cudaStream_t);
CZC_G4_INST(float)
CZC_G4_INST(double)
#undef CZC_G4_INST

}  // namespace czc

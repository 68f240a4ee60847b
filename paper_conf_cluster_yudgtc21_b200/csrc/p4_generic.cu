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
deriv4_kernel(Field4<T> s, double* __restrict__ parts, DevResults* __restrict__ res, unsigned int* __restrict__ ticket) {
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

// Local SSIM of every window of the grid, one window per thread step: FP64 sums of the moments
// a = x - K, e = y - x, a (y - K), e^2 anchored at the window's first original sample K (the
// cancellation is bounded by the window's own range), exact min / max of x, then the mix of the
// 3-D engine (cancellation-free two-factor form, reading R14 / R15).
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
    double sa = 0, se = 0, sab = 0, see = 0;
    T mn = s.x[o], mx = mn;
    for (int l = 0; l < p.w[0]; l++)
      for (int k = 0; k < p.w[1]; k++)
        for (int j = 0; j < p.w[2]; j++) {
          const int64_t r = o + l * s.st[0] + k * s.st[1] + j * s.st[2];
          for (int q = 0; q < p.w[3]; q++) {
            const T xv = __ldg(s.x + r + q), yv = __ldg(s.y + r + q);
            const double xd = xv, yd = yv;
            const double a = xd - K, b = yd - K, e = yd - xd;
            sa += a; se += e; sab = fma(a, b, sab); see = fma(e, e, see);
            mn = tmin(mn, xv);
            mx = tmax(mx, xv);
          }
        }
    const double mua = sa * invM, mue = se * invM;
    const double mux = K + mua, muy = mux + mue;
    const double sxy = sab * invM - mua * (mua + mue);
    const double sv = see * invM - mue * mue;
    double L = p.range_mode ? Lglob : (double)mx - (double)mn;
    L = (L == 0.0) ? 1.0 : L;
    const double C1 = (0.01 * L) * (0.01 * L), C2 = (0.03 * L) * (0.03 * L);
    const double A = 2.0 * mux * muy + C1, B = 2.0 * sxy + C2;
    const double ssim = (A * B) / ((A + mue * mue) * (B + sv));
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

// Step 1 along axis 2 (the common case): a thread takes a run of kRun4 consecutive axis-2
// origins and slides along that axis — per window one new slab of w0 w1 w3 samples enters and
// one leaves (recomputed: no per-thread sums ring), instead of w0 w1 w2 w3 samples per window.
// Adjacent threads take adjacent x-origins (x stays the fastest index), so every load of a warp
// is coalesced and neighbouring windows share L1 lines.  The slab extrema of the last w2 slabs
// sit in a per-thread shared-memory ring; the moments are anchored at the run's first sample.
constexpr int kRun4 = 16;
constexpr int kRunThreads = 128;                   // the extrema ring: 16 x 128 x 2 x sizeof(T)
template <typename T>
__device__ __forceinline__ void slab4(const Field4<T>& s, int64_t base, const int w[4], double K, double& sa,
                                      double& se, double& sab, double& see, T& mn, T& mx) {
  sa = se = sab = see = 0;
  mn = s.x[base];
  mx = mn;
  for (int l = 0; l < w[0]; l++)
    for (int k = 0; k < w[1]; k++) {
      const int64_t r = base + l * s.st[0] + k * s.st[1];
      for (int q = 0; q < w[3]; q++) {
        const T xv = __ldg(s.x + r + q), yv = __ldg(s.y + r + q);
        const double xd = xv, yd = yv;
        const double a = xd - K, b = yd - K, e = yd - xd;
        sa += a; se += e; sab = fma(a, b, sab); see = fma(e, e, see);
        mn = tmin(mn, xv);
        mx = tmax(mx, xv);
      }
    }
}

template <typename T>
__global__ void __launch_bounds__(kRunThreads)
ssim4_run_kernel(Field4<T> s, Ssim4Params p, double* __restrict__ parts, DevResults* __restrict__ res,
                 unsigned int* __restrict__ ticket, double* __restrict__ dbg) {
  __shared__ T ring_mn[16][kRunThreads], ring_mx[16][kRunThreads];   // w2 <= 16 (kMaxWin)
  const double Lglob = res->p1g.xmax - res->p1g.xmin;
  const double invM = 1.0 / (double)(p.w[0] * p.w[1] * p.w[2] * p.w[3]);
  const int w2 = p.w[2];
  const int64_t nr = (p.nw[2] + kRun4 - 1) / kRun4;             // runs along axis 2
  const int64_t lenr[4] = {p.nw[0], p.nw[1], nr, p.nw[3]};
  const int64_t total = lenr[0] * lenr[1] * lenr[2] * lenr[3];
  const int t = threadIdx.x;
  double ssum = 0, scnt = 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + t; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t c4[4];
    decode4(i, lenr, c4);
    const int64_t r0 = c4[2] * kRun4;
    const int64_t r1 = min(r0 + kRun4, p.nw[2]);                // axis-2 origins [r0, r1)
    const int64_t base = c4[0] * p.s[0] * s.st[0] + c4[1] * p.s[1] * s.st[1] + c4[3] * p.s[3];
    const double K = s.x[base + r0 * s.st[2]];
    double Sa = 0, Se = 0, Sab = 0, See = 0;
    for (int q = 0; q < w2; q++) {                               // the first window's slabs
      double a, e, ab, ee;
      T mn, mx;
      slab4(s, base + (r0 + q) * s.st[2], p.w, K, a, e, ab, ee, mn, mx);
      Sa += a; Se += e; Sab += ab; See += ee;
      ring_mn[q][t] = mn;
      ring_mx[q][t] = mx;
    }
    for (int64_t o = r0; o < r1; o++) {
      if (o > r0) {                                              // slide: slab o+w2-1 in, o-1 out
        double a, e, ab, ee, ao, eo, abo, eeo;
        T mn, mx, mno, mxo;
        slab4(s, base + (o + w2 - 1) * s.st[2], p.w, K, a, e, ab, ee, mn, mx);
        slab4(s, base + (o - 1) * s.st[2], p.w, K, ao, eo, abo, eeo, mno, mxo);
        Sa += a - ao; Se += e - eo; Sab += ab - abo; See += ee - eeo;
        const int slot = (int)((o - r0 + w2 - 1) % 16);
        ring_mn[slot][t] = mn;
        ring_mx[slot][t] = mx;
      }
      T wmn = ring_mn[(o - r0) % 16][t], wmx = ring_mx[(o - r0) % 16][t];
      for (int q = 1; q < w2; q++) {
        const int slot = (int)((o - r0 + q) % 16);
        wmn = tmin(wmn, ring_mn[slot][t]);
        wmx = tmax(wmx, ring_mx[slot][t]);
      }
      const double mua = Sa * invM, mue = Se * invM;
      const double mux = K + mua, muy = mux + mue;
      const double sxy = Sab * invM - mua * (mua + mue);
      const double sv = See * invM - mue * mue;
      double L = p.range_mode ? Lglob : (double)wmx - (double)wmn;
      L = (L == 0.0) ? 1.0 : L;
      const double C1 = (0.01 * L) * (0.01 * L), C2 = (0.03 * L) * (0.03 * L);
      const double A = 2.0 * mux * muy + C1, B = 2.0 * sxy + C2;
      const double ssim = (A * B) / ((A + mue * mue) * (B + sv));
      ssum += ssim;
      scnt += 1.0;
      if (dbg) dbg[((c4[0] * p.nw[1] + c4[1]) * p.nw[2] + o) * p.nw[3] + c4[3]] = ssim;
    }
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
                          unsigned int* ticket, cudaStream_t st) {
  const Field4<T> f = field4(x, y, n);
  const int64_t nI = (n[0] - 2) * (n[1] - 2) * (n[2] - 2) * (n[3] - 2);
  deriv4_kernel<T><<<g4_grid(nI, sms), kG4Threads, 0, st>>>(f, parts, res, ticket);
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
  if (p.s[2] == 1 && p.w[2] <= 16) {
    const int64_t runs = total / p.nw[2] * ((p.nw[2] + kRun4 - 1) / kRun4);
    int64_t b = (runs + kRunThreads - 1) / kRunThreads;
    if (b > g4_max_blocks(sms)) b = g4_max_blocks(sms);
    ssim4_run_kernel<T><<<(unsigned)(b < 1 ? 1 : b), kRunThreads, 0, st>>>(f, p, parts, res, ticket, dbg);
  }
  else
    ssim4_kernel<T><<<g4_grid(total, sms), kG4Threads, 0, st>>>(f, p, parts, res, ticket, dbg);
  return cudaGetLastError();
}

#define CZC_G4_INST(T)                                                                                         \
  template cudaError_t launch_deriv4<T>(const T*, const T*, const int64_t*, int, double*, DevResults*,         \
                                        unsigned int*, cudaStream_t);                                          \
  template cudaError_t launch_ac4<T>(const T*, const T*, const int64_t*, int, int, double*, DevResults*,       \
                                     unsigned int*, cudaStream_t);                                             \
  template cudaError_t launch_ssim4<T>(const T*, const T*, const int64_t*, const int*, const int*, int, int,   \
                                       double*, DevResults*, unsigned int*, double*, cudaStream_t);
CZC_G4_INST(float)
CZC_G4_INST(double)
#undef CZC_G4_INST

}  // namespace czc

// p1_reduce.cu — Pattern 1: fused global reduction over the (orig, recon) pair.
//
// Paper: Table I Category I (L107) — min/max/avg error, pwr error, MSE, RMSE, NRMSE, SNR, PSNR;
// "one data read from global memory to registers can feed two reductions" (L118); Alg. 1
// (L173-L203): per-thread strided reduce -> warp shuffles -> shared memory -> per-block partial
// -> grid-level reduction.  B200 design: a persistent grid of 148 x k blocks
// streams both arrays with 128-bit L1-bypassing loads; every element feeds all P1 statistics at
// once; the per-block partials are combined by the last block to finish, in block-index order
// (deterministic, no float atomics, no cooperative grid sync — reading R18).
#include "czc_internal.cuh"

namespace czc {

// 32: 256-bit float32 vectors (LDG.E.ENL2.256).  Not the default: at two vectors in flight per
// array they need 162 registers (one block per SM) or spill 120 B at two blocks per SM, and one
// 256-bit vector in flight carries the same bytes as the two 128-bit ones of the default.
#ifndef CZC_P1_VEC_BYTES
#define CZC_P1_VEC_BYTES 16
#endif
constexpr int kP1VecBytes = CZC_P1_VEC_BYTES;

// Per-thread accumulator: sums about the thread's first element (kx, ke).  The element count
// is implicit (counted per vector), so no per-element work is spent on it.

template <typename T>
struct P1Acc {
  double kx, ke;
  double sa, sc, saa, sac, scc, sae;   // d_a = x - kx, d_c = e - ke (d_b = y - (kx + ke) = d_a + d_c)
  double emin, emax, pmin, pmax, spwr;
  double pthr_hi, pthr_lo;          // candidate thresholds for the exact pwr extrema
  unsigned npwr;                    // count of x != 0 (per thread, < 2^32)
  T xmin, xmax;                     // exact, in the input type
};

template <typename T>
__device__ __forceinline__ void acc_init(P1Acc<T>& a, T kxf, T kyf) {
  a.kx = kxf; a.ke = (double)kyf - (double)kxf;
  a.sa = a.sc = a.saa = a.sac = a.scc = a.sae = 0;
  a.emin = dinf(); a.emax = -dinf(); a.pmin = dinf(); a.pmax = -dinf(); a.spwr = 0;
  a.pthr_hi = -dinf(); a.pthr_lo = dinf();
  a.npwr = 0;
  a.xmin = (T)dinf(); a.xmax = -(T)dinf();
}


// One element: e = recon - orig in double (reading R1; same rounding as the oracle).  Point-wise
// relative error |e|/|x| (reading R3): its SUM uses q~ = |e| * r, r = rcp.approx(|x|) refined by
// one Newton step (relative error of q~ < 1e-12: measured max 8.6e-13 for r, profiles/
// r01_rcp_probe.txt; far inside the 1e-9 tolerance of pwr_mean); its extrema must be the IEEE
// quotient, bit-exact with the oracle, so the correctly rounded division runs only for
// candidates: an element can raise the maximum only if q~ > thr_hi = pmax (1 - 1e-10) (q~ >=
// Q (1 - 1e-12) and pmax <= RN(Q) for a larger true quotient Q), and lower the minimum only if
// q~ < thr_lo = pmin (1 + 1e-10); a zero minimum admits no further candidate (thr_lo = 0), a zero
// maximum admits only q~ > 0.  Returns whether this element is a candidate; candidates are
// resolved per vector, warp-uniformly (see acc_vec).  float64 inputs: e = y - x is rounded to
// double exactly as in the oracle (R1), and |x| outside [1e-290, 1e290] (where the approximate
// reciprocal flushes) takes the IEEE quotient.
template <typename T>
__device__ __forceinline__ bool acc_elem(P1Acc<T>& a, T xf, T yf, double& ae_out, double& ax_out) {
  const double x = xf, y = yf;
  const double e = y - x;
  // y - (kx + ke) = (x - kx) + (e - ke): the recon moments follow from d_a, d_c and their cross
  // sum (6 accumulators instead of 8)
  const double da = x - a.kx, dc = e - a.ke;
  a.sa += da; a.sc += dc;
  a.saa = fma(da, da, a.saa);
  a.sac = fma(da, dc, a.sac);
  a.scc = fma(dc, dc, a.scc);
  const double ae = fabs(e);
  a.sae += ae;
  a.emin = e < a.emin ? e : a.emin;
  a.emax = e > a.emax ? e : a.emax;
  a.xmin = tmin(a.xmin, xf);
  a.xmax = tmax(a.xmax, xf);
  const bool nz = xf != (T)0;
  const double ax = nz ? fabs(x) : 1.0;
  // |e| = |x| (a reconstruction of 0 or 2x: common where a relative error bound exceeds the
  // value, e.g. the low decades of a log-normal density) gives exactly 1 — and would otherwise
  // be a candidate on every such element once the maximum is 1 (a tie the approximate quotient
  // cannot rule out): C3 P1 ran at 29 % of HBM
  const bool unit = ae == ax;
  double qa = nz ? (unit ? 1.0 : ae * rcp_newton1(ax)) : 0.0;
  if (sizeof(T) == 8 && !(ax >= 1e-290 && ax <= 1e290)) qa = ae / ax;
  a.spwr += qa;
  a.npwr += nz ? 1u : 0u;
  ae_out = ae;
  ax_out = ax;
  return nz && (unit ? (1.0 > a.pmax || 1.0 < a.pmin) : (qa > a.pthr_hi || qa < a.pthr_lo));
}

template <typename T>
__device__ __forceinline__ void acc_resolve(P1Acc<T>& a, double ae, double ax) {
  const double q = ae / ax;                          // IEEE, correctly rounded
  if (q > a.pmax) { a.pmax = q; a.pthr_hi = q * (1.0 - 1e-10); }
  if (q < a.pmin) { a.pmin = q; a.pthr_lo = q * (1.0 + 1e-10); }   // q = 0 -> thr_lo = 0
}

// One vector of VB bytes of the input type (16: 4 floats / 2 doubles; 32: 8 floats, one 256-bit
// LDG.E.ENL2.256 per array).
template <typename T, int VB>
struct VecB {
  static constexpr int N = VB / (int)sizeof(T);
  T e[N];
};
template <typename T, int VB>
__device__ __forceinline__ VecB<T, VB> ld_streamB(const T* p) {
  VecB<T, VB> r;
  if constexpr (VB == 32 && sizeof(T) == 4) {
    asm volatile("ld.global.nc.L1::no_allocate.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=f"(r.e[0]), "=f"(r.e[1]), "=f"(r.e[2]), "=f"(r.e[3]), "=f"(r.e[4]), "=f"(r.e[5]),
                   "=f"(r.e[6]), "=f"(r.e[7]) : "l"(p));
  } else {
    static_assert(VB == 16, "256-bit loads: float32 only");
    const Vec16<T> v = ld_stream16(p);
#pragma unroll
    for (int j = 0; j < VecB<T, VB>::N; j++) r.e[j] = v.e[j];
  }
  return r;
}

template <typename T, int VB>
__device__ __forceinline__ void acc_vec(P1Acc<T>& a, const VecB<T, VB>& xv, const VecB<T, VB>& yv) {
  constexpr int N = VecB<T, VB>::N;
  double ae[N], ax[N];
  bool c[N], any = false;
#pragma unroll
  for (int j = 0; j < N; j++) {
    c[j] = acc_elem(a, xv.e[j], yv.e[j], ae[j], ax[j]);
    any |= c[j];
  }
  // Warp-uniform resolve; in a full warp the lanes then share their extrema (a lane may report
  // the warp's maximum / minimum: merging takes max / min, so the result is unchanged), which
  // makes later candidates ~32x rarer than with per-lane thresholds.
  const unsigned m = __activemask();
  if (__any_sync(m, any)) {
#pragma unroll
    for (int j = 0; j < N; j++)
      if (c[j]) acc_resolve(a, ae[j], ax[j]);
    if (m == 0xffffffffu) {
      double mx = a.pmax, mn = a.pmin;
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) {
        const double ox = __shfl_xor_sync(m, mx, off), on = __shfl_xor_sync(m, mn, off);
        mx = ox > mx ? ox : mx;
        mn = on < mn ? on : mn;
      }
      if (mx > a.pmax) { a.pmax = mx; a.pthr_hi = mx * (1.0 - 1e-10); }
      if (mn < a.pmin) { a.pmin = mn; a.pthr_lo = mn * (1.0 + 1e-10); }
    }
  }
}

template <typename T>
__device__ __forceinline__ void acc_scalar(P1Acc<T>& a, T xf, T yf) {
  double ae, ax;
  if (acc_elem(a, xf, yf, ae, ax)) acc_resolve(a, ae, ax);
}

template <typename T>
__device__ __forceinline__ P1State acc_to_state(const P1Acc<T>& a, double n) {
  P1State s;
  p1_empty(s);
  s.sae = a.sae; s.spwr = a.spwr; s.npwr = (double)a.npwr;
  s.emin = a.emin; s.emax = a.emax; s.pmin = a.pmin; s.pmax = a.pmax;
  s.xmin = a.xmin; s.xmax = a.xmax;
  if (n > 0) {
    s.n = n;
    s.mx = a.kx + a.sa / n;
    const double sb = a.sa + a.sc, sbb = a.saa + 2.0 * a.sac + a.scc, sab = a.saa + a.sac;
    s.my = (a.kx + a.ke) + sb / n;
    s.me = a.ke + a.sc / n;
    s.m2x = a.saa - a.sa * (a.sa / n);
    s.m2y = sbb - sb * (sb / n);
    s.cxy = sab - a.sa * (sb / n);
    s.m2e = a.scc - a.sc * (a.sc / n);
  }
  return s;
}

__device__ __forceinline__ P1State shfl_down_state(const P1State& s, int off) {
  P1State r;
  const int* src = reinterpret_cast<const int*>(&s);
  int* dst = reinterpret_cast<int*>(&r);
#pragma unroll
  for (int i = 0; i < kP1Words; i++) dst[i] = __shfl_down_sync(0xffffffffu, src[i], off);
  return r;
}

// Merge the block's per-thread states in a fixed tree; result valid in thread 0.
__device__ __forceinline__ P1State block_merge(P1State s) {
  __shared__ P1State s_w[32];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
  for (int off = 16; off > 0; off >>= 1) {
    P1State o = shfl_down_state(s, off);
    if (lane + off < 32) p1_merge(s, o);
  }
  if (lane == 0) s_w[warp] = s;
  __syncthreads();
  if (warp == 0) {
    if (lane < nw) s = s_w[lane]; else p1_empty(s);
    for (int off = 16; off > 0; off >>= 1) {
      P1State o = shfl_down_state(s, off);
      if (lane + off < 32) p1_merge(s, o);
    }
  }
  __syncthreads();
  return s;
}

// VEC: x and y share the same 16-byte misalignment; elements [head, head + VN*nvec) are read as
// 128-bit vectors (VN = 4 floats or 2 doubles), the leftovers (prologue [0, head) and tail) by
// threads 0..nleft-1.
template <typename T, bool VEC, int VB>
__global__ void __launch_bounds__(kP1Threads)
p1_kernel(const T* __restrict__ x, const T* __restrict__ y, int64_t n, int64_t head,
          P1State* __restrict__ parts, DevResults* __restrict__ res, unsigned int* __restrict__ ticket) {
  constexpr int VN = VecB<T, VB>::N;
  const int64_t gtid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t gsz = (int64_t)gridDim.x * blockDim.x;
  const int64_t nvec = VEC ? (n - head) / VN : 0;
  const int64_t tail0 = head + VN * nvec;
  const int64_t nleft = VEC ? head + (n - tail0) : n;   // scalar elements
  auto left_index = [&](int64_t k) -> int64_t { return VEC ? (k < head ? k : tail0 + (k - head)) : k; };

  P1Acc<T> a;
  int64_t first = -1;   // anchor = the thread's first element
  if (VEC && gtid < nvec) first = head + VN * gtid;
  else if (gtid < nleft) first = left_index(gtid);
  acc_init(a, first >= 0 ? x[first] : (T)0, first >= 0 ? y[first] : (T)0);

  int64_t cnt = 0;                                 // elements processed by this thread
  if (VEC) {
    const T* x4 = x + head;
    const T* y4 = y + head;
    int64_t v = gtid;
    if (gtid < nvec) cnt = VN * ((nvec - 1 - gtid) / gsz + 1);
    // software pipeline: the next two vectors' loads are in flight while two are processed
    if (v + gsz < nvec) {
      VecB<T, VB> xa = ld_streamB<T, VB>(x4 + VN * v), ya = ld_streamB<T, VB>(y4 + VN * v);
      VecB<T, VB> xb = ld_streamB<T, VB>(x4 + VN * (v + gsz)), yb = ld_streamB<T, VB>(y4 + VN * (v + gsz));
      v += 2 * gsz;
      for (; v + gsz < nvec; v += 2 * gsz) {
        const VecB<T, VB> xc = ld_streamB<T, VB>(x4 + VN * v), yc = ld_streamB<T, VB>(y4 + VN * v);
        const VecB<T, VB> xd = ld_streamB<T, VB>(x4 + VN * (v + gsz)), yd = ld_streamB<T, VB>(y4 + VN * (v + gsz));
        acc_vec<T, VB>(a, xa, ya);
        acc_vec<T, VB>(a, xb, yb);
        xa = xc; ya = yc; xb = xd; yb = yd;
      }
      acc_vec<T, VB>(a, xa, ya);
      acc_vec<T, VB>(a, xb, yb);
    }
    for (; v < nvec; v += gsz) acc_vec<T, VB>(a, ld_streamB<T, VB>(x4 + VN * v), ld_streamB<T, VB>(y4 + VN * v));
    if (gtid < nleft) {
      const int64_t i = left_index(gtid);
      acc_scalar(a, x[i], y[i]);
      cnt += 1;
    }
  } else {
    if (gtid < n) cnt = (n - 1 - gtid) / gsz + 1;
    for (int64_t i = gtid; i < n; i += gsz) acc_scalar(a, x[i], y[i]);
  }

  P1State s = block_merge(acc_to_state(a, (double)cnt));
  if (threadIdx.x == 0) parts[blockIdx.x] = s;
  if (!last_block_arrive(ticket)) return;

  // Last block: fold the partials in block-index order (thread t: t, t+T, ...), fixed tree.
  P1State f;
  p1_empty(f);
  for (int b = threadIdx.x; b < (int)gridDim.x; b += blockDim.x) {
    P1State pb;
    const double* src = reinterpret_cast<const double*>(parts + b);
    double* dst = reinterpret_cast<double*>(&pb);
#pragma unroll
    for (int i = 0; i < (int)(sizeof(P1State) / 8); i++) dst[i] = __ldcg(src + i);
    p1_merge(f, pb);
  }
  f = block_merge(f);
  if (threadIdx.x == 0) {
    res->rec.p1 = f;
    res->p1g = f;
    *ticket = 0;   // re-arm for the next launch
  }
}

// Vector path: both arrays element-aligned with the same VB-byte misalignment; head = elements
// before the first aligned vector.
template <typename T, int VB>
static bool vec_head(const T* x, const T* y, int64_t n, int64_t* head) {
  const uintptr_t ax = reinterpret_cast<uintptr_t>(x), ay = reinterpret_cast<uintptr_t>(y);
  const bool vec = (ax % VB) == (ay % VB) && (ax % sizeof(T)) == 0;
  int64_t h = vec ? (int64_t)(((VB - ax % VB) % VB) / sizeof(T)) : 0;
  *head = h > n ? n : h;
  return vec;
}

// Host launcher.  Returns the cuda error of the launch.  float32 pairs with the same 32-byte
// misalignment stream 256-bit vectors (twice the bytes in flight per load instruction), others
// 128-bit vectors, else scalars.
template <typename T>
cudaError_t launch_p1(const T* x, const T* y, int64_t n, int grid_cap, P1State* parts,
                      DevResults* res, unsigned int* ticket, cudaStream_t st) {
  int64_t head = 0;
  auto grid = [&](int64_t work) {
    int64_t blocks = (work + kP1Threads - 1) / kP1Threads;
    if (blocks > grid_cap) blocks = grid_cap;
    return (unsigned)(blocks < 1 ? 1 : blocks);
  };
  if constexpr (sizeof(T) == 4 && kP1VecBytes == 32) {
    if (vec_head<T, 32>(x, y, n, &head)) {
      p1_kernel<T, true, 32><<<grid((n - head) / 8 + 8), kP1Threads, 0, st>>>(x, y, n, head, parts, res, ticket);
      return cudaGetLastError();
    }
  }
  if (vec_head<T, 16>(x, y, n, &head))
    p1_kernel<T, true, 16><<<grid((n - head) / Vec16<T>::N + 8), kP1Threads, 0, st>>>(x, y, n, head, parts, res, ticket);
  else
    p1_kernel<T, false, 16><<<grid(n), kP1Threads, 0, st>>>(x, y, n, head, parts, res, ticket);
  return cudaGetLastError();
}
template cudaError_t launch_p1<float>(const float*, const float*, int64_t, int, P1State*, DevResults*,
                                      unsigned int*, cudaStream_t);
template cudaError_t launch_p1<double>(const double*, const double*, int64_t, int, P1State*, DevResults*,
                                       unsigned int*, cudaStream_t);

// ------------------------------------------------------------------------------------------------
// Error PDF / pwr-error PDF (Table I Category I, L107; reading R24).  One pass after P1: the bins
// span the GLOBAL extrema found by P1 (res->p1g), so the counts need no second scan.  Every block
// keeps a shared-memory histogram of 32-bit counters and folds it into the 64-bit device counts
// with one global atomicAdd per non-empty bin (integer sums: order-independent, deterministic).
// Bin index: fast path q = (v - lo) * (1/w); when q lies within a relative 1e-10 of a bin edge,
// the IEEE quotient (v - lo) / w decides (|q - RN((v - lo) / w)| <= ~2 ulp of q), so every count
// is bit-exact with the oracle's floor((v - lo) / w).  The pwr value is |e| * rcp(|x|) (relative
// error < 1e-12, see acc_elem); near an edge the IEEE |e| / |x| is formed first.
// ------------------------------------------------------------------------------------------------
__device__ __forceinline__ int pdf_clamp(double q, int nb) {
  const int b = (int)floor(q);
  return b >= nb ? nb - 1 : (b < 0 ? 0 : b);
}
__device__ __forceinline__ bool pdf_near_edge(double q, double tol) {
  const double f = floor(q);
  return q - f < tol || f + 1.0 - q < tol;
}
__device__ __forceinline__ int pdf_bin_err(double e, const PdfRange& r) {
  if (!(r.rw > 0)) return 0;
  const double q = (e - r.lo) * r.rw;                 // e >= lo
  if (pdf_near_edge(q, 1e-10 * (q + 1.0))) return pdf_clamp((e - r.lo) / r.w, r.nb);
  return pdf_clamp(q, r.nb);
}
__device__ __forceinline__ int pdf_bin_pwr(double ae, double ax, const PdfRange& r) {
  if (!(r.rw > 0)) return 0;
  double qa = ae * rcp_newton1(ax);
  if (!(ax >= 1e-290 && ax <= 1e290)) qa = ae / ax;         // float64 inputs only
  const double t = (qa - r.lo) * r.rw;
  if (pdf_near_edge(t, 1e-10 * (fabs(qa) * r.rw + 1.0))) return pdf_clamp((ae / ax - r.lo) / r.w, r.nb);
  return pdf_clamp(t, r.nb);
}

template <typename T, bool VEC>
__global__ void __launch_bounds__(kP1Threads)
pdf_kernel(const T* __restrict__ x, const T* __restrict__ y, int64_t n, int64_t head, int nb,
           DevResults* __restrict__ res) {
  constexpr int VN = Vec16<T>::N;
  __shared__ unsigned int h[2][CZC_PDF_MAX_BINS];
  for (int i = threadIdx.x; i < 2 * CZC_PDF_MAX_BINS; i += blockDim.x) (&h[0][0])[i] = 0u;
  __syncthreads();
  const P1State& g = res->p1g;
  const PdfRange re = pdf_range(g.emin, g.emax, nb);
  const PdfRange rp = pdf_range(g.pmin, g.pmax, nb);
  auto elem = [&](T xf, T yf) {
    const double xd = xf, e = (double)yf - xd;
    atomicAdd(&h[0][pdf_bin_err(e, re)], 1u);
    if (xf != (T)0) atomicAdd(&h[1][pdf_bin_pwr(fabs(e), fabs(xd), rp)], 1u);
  };
  const int64_t gtid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t gsz = (int64_t)gridDim.x * blockDim.x;
  if (VEC) {
    const int64_t nvec = (n - head) / VN, tail0 = head + VN * nvec;
    for (int64_t v = gtid; v < nvec; v += gsz) {
      const Vec16<T> a = ld_stream16(x + head + VN * v), b = ld_stream16(y + head + VN * v);
#pragma unroll
      for (int j = 0; j < VN; j++) elem(a.e[j], b.e[j]);
    }
    if (gtid < head) elem(x[gtid], y[gtid]);
    if (gtid < n - tail0) elem(x[tail0 + gtid], y[tail0 + gtid]);
  } else {
    for (int64_t i = gtid; i < n; i += gsz) elem(x[i], y[i]);
  }
  __syncthreads();
  unsigned long long* out = &res->rec.pdf[0][0];
  for (int i = threadIdx.x; i < nb; i += blockDim.x) {
    if (h[0][i]) atomicAdd(out + i, (unsigned long long)h[0][i]);
    if (h[1][i]) atomicAdd(out + CZC_PDF_MAX_BINS + i, (unsigned long long)h[1][i]);
  }
}

// Zeroes the counts, then histograms x[0, n), y[0, n) into res->rec.pdf (needs res->p1g).
template <typename T>
cudaError_t launch_pdf(const T* x, const T* y, int64_t n, int nb, int grid_cap, DevResults* res,
                       cudaStream_t st) {
  cudaError_t e = cudaMemsetAsync(res->rec.pdf, 0, sizeof(res->rec.pdf), st);
  if (e != cudaSuccess) return e;
  int64_t head = 0;
  const bool vec = vec_head<T, 16>(x, y, n, &head);
  const int64_t work = vec ? ((n - head) / Vec16<T>::N + 8) : n;
  int64_t blocks = (work + kP1Threads - 1) / kP1Threads;
  if (blocks > grid_cap) blocks = grid_cap;
  if (blocks < 1) blocks = 1;
  if (vec) pdf_kernel<T, true><<<(unsigned)blocks, kP1Threads, 0, st>>>(x, y, n, head, nb, res);
  else pdf_kernel<T, false><<<(unsigned)blocks, kP1Threads, 0, st>>>(x, y, n, head, nb, res);
  return cudaGetLastError();
}
template cudaError_t launch_pdf<float>(const float*, const float*, int64_t, int, int, DevResults*, cudaStream_t);
template cudaError_t launch_pdf<double>(const double*, const double*, int64_t, int, int, DevResults*, cudaStream_t);

// Slab mode: merge the allgathered per-rank states in rank order (every rank runs the same code
// on the same bytes, so all ranks hold identical results).
__global__ void p1_combine_kernel(const P1State* __restrict__ states, int count, DevResults* __restrict__ res) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  P1State f;
  p1_empty(f);
  for (int r = 0; r < count; r++) p1_merge(f, states[r]);
  res->p1g = f;
}

cudaError_t launch_p1_combine(const P1State* states, int count, DevResults* res, cudaStream_t st) {
  p1_combine_kernel<<<1, 32, 0, st>>>(states, count, res);
  return cudaGetLastError();
}

int p1_max_blocks_per_sm() {
  int nb = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, p1_kernel<float, true, kP1VecBytes>, kP1Threads, 0);
  return nb > 0 ? nb : 1;
}

}  // namespace czc

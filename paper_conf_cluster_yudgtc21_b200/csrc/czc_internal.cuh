// czc_internal.cuh — shared device/host definitions of the CUDA path (never used by oracle/).
//
// Partial-result records, the order-fixed (deterministic) cross-block finish, and small device
// helpers.  Citations "Lnnn" are PAPER.md lines; DESIGN.md §5 describes the kernels.
#pragma once
#include <atomic>

#include <cuda_runtime.h>
#include <stdint.h>
#include <stddef.h>
#include <string.h>

#include "../../include/czc.h"

// host/device bit casts
__host__ __device__ inline double czc_bits_to_double(long long v) {
#if defined(__CUDA_ARCH__)
  return __longlong_as_double(v);
#else
  double d;
  memcpy(&d, &v, 8);
  return d;
#endif
}
__host__ __device__ inline float czc_bits_to_float(int v) {
#if defined(__CUDA_ARCH__)
  return __int_as_float(v);
#else
  float f;
  memcpy(&f, &v, 4);
  return f;
#endif
}

namespace czc {

constexpr int kMaxWin = 16;      // largest SSIM window extent per axis on the fast path
constexpr int kP1Threads = 256;
constexpr int kFinishThreads = 256;

__host__ __device__ inline double dinf() { return czc_bits_to_double(0x7ff0000000000000ll); }
__host__ __device__ inline float finf() { return czc_bits_to_float(0x7f800000); }

// ------------------------------------------------------------------------------------------------
// P1 state in merge ("Chan") form: counts, means and centred co-moments.  Per-thread sums are
// taken about the thread's first element (so the shifted-sum cancellation is bounded by the
// thread's element count), converted to centred form once, and then merged pairwise with the
// numerically stable update  M2 = M2a + M2b + d^2 na nb / n  (no catastrophic cancellation).
// Fields map to Table I Category I (L107) and the north_star list; see DESIGN.md §5.1.
// ------------------------------------------------------------------------------------------------
struct P1State {
  double n;                   // element count (exact as double below 2^53)
  double mx, my, me;          // means of x, y, e = y - x
  double m2x, m2y, cxy, m2e;  // sum (x-mx)^2, sum (y-my)^2, sum (x-mx)(y-my), sum (e-me)^2
  double sae;                 // sum |e|
  double emin, emax;          // extrema of e (exact doubles)
  double pmin, pmax, spwr;    // point-wise relative error |e|/|x| over x != 0
  double npwr;                // count of x != 0
  double xmin, xmax;          // extrema of x (exact: float32 and float64 samples are doubles)
};
constexpr int kP1Words = sizeof(P1State) / 4;
static_assert(sizeof(P1State) % 8 == 0, "P1State must be a whole number of doubles");

__host__ __device__ inline void p1_empty(P1State& s) {
  s.n = 0; s.mx = s.my = s.me = 0; s.m2x = s.m2y = s.cxy = s.m2e = 0; s.sae = 0;
  s.emin = dinf(); s.emax = -dinf();
  s.pmin = dinf(); s.pmax = -dinf(); s.spwr = 0; s.npwr = 0;
  s.xmin = dinf(); s.xmax = -dinf();
}

__host__ __device__ inline void p1_merge(P1State& a, const P1State& b) {
  a.sae += b.sae; a.spwr += b.spwr; a.npwr += b.npwr;
  a.emin = b.emin < a.emin ? b.emin : a.emin;
  a.emax = b.emax > a.emax ? b.emax : a.emax;
  a.pmin = b.pmin < a.pmin ? b.pmin : a.pmin;
  a.pmax = b.pmax > a.pmax ? b.pmax : a.pmax;
  a.xmin = b.xmin < a.xmin ? b.xmin : a.xmin;
  a.xmax = b.xmax > a.xmax ? b.xmax : a.xmax;
  if (b.n == 0) return;
  if (a.n == 0) {
    a.n = b.n; a.mx = b.mx; a.my = b.my; a.me = b.me;
    a.m2x = b.m2x; a.m2y = b.m2y; a.cxy = b.cxy; a.m2e = b.m2e;
    return;
  }
  const double n = a.n + b.n, fb = b.n / n, g = a.n * fb;
  const double dx = b.mx - a.mx, dy = b.my - a.my, de = b.me - a.me;
  a.mx += dx * fb; a.my += dy * fb; a.me += de * fb;
  a.m2x += b.m2x + dx * dx * g;
  a.m2y += b.m2y + dy * dy * g;
  a.cxy += b.cxy + dx * dy * g;
  a.m2e += b.m2e + de * de * g;
  a.n = n;
}

// ------------------------------------------------------------------------------------------------
// Slot-wise partial records for P2 / P3: each block writes K doubles; the finish combines slot k
// with its op (sum / min / max) in a fixed order, independent of block completion order.
// ------------------------------------------------------------------------------------------------
enum : int { OP_SUM = 0, OP_MIN = 1, OP_MAX = 2 };

// Derivative record: per field f (5): [max|dF|, sum|dF|, sum dF^2, min F(x), max F(x)]
constexpr int kDerivStats = 5;
constexpr int kDerivSlots = kDerivStats * CZC_NDERIV;
__host__ __device__ constexpr int deriv_op(int slot) {
  return (slot % kDerivStats) == 0 ? OP_MAX : (slot % kDerivStats) == 3 ? OP_MIN
       : (slot % kDerivStats) == 4 ? OP_MAX : OP_SUM;
}
// Autocorrelation record: S(tau) for tau = 1..CZC_MAX_LAG (index tau-1), all sums; one record
// per walk axis (z, y, x), summed at the finish.
constexpr int kAcSlots = CZC_MAX_LAG;
constexpr int kAcWalks = 3;
// SSIM record: [sum of local SSIM, number of windows, windows recomputed exactly]
constexpr int kSsimSlots = 3;

// The partial-result record of one field (or one slab of it): what one rank contributes and what
// the rank-ordered combine consumes (czc_combine).  Layout is internal, size = czc_sizeof(3).
struct Record {
  P1State p1;                        // this field's / slab's own P1 state
  double deriv[kDerivSlots];
  double ac[kAcWalks][kAcSlots];
  double ssim[kSsimSlots];
  unsigned long long pdf[2][CZC_PDF_MAX_BINS];   // error / pwr-error PDF counts (CZC_M_PDF); last
};
// bytes of a Record that carry results when no PDF was requested (the D2H copy stops there)
constexpr size_t kRecordNoPdf = offsetof(Record, pdf);

// PDF bin of v (reading R24; the oracle implements the same definition): equal-width bins of
// width w = (hi - lo) / nb starting at lo, b = floor((v - lo) / w) in IEEE double with the top
// edge clamped into the last bin; w == 0 (all values equal) or a non-finite w gives bin 0.
struct PdfRange {
  double lo, w, rw;                  // rw = 1 / w (IEEE), for the fast path
  int nb;
};
__host__ __device__ inline PdfRange pdf_range(double lo, double hi, int nb) {
  PdfRange r;
  r.lo = lo;
  r.nb = nb;
  r.w = (hi - lo) / (double)nb;
  r.rw = r.w > 0 && r.w < dinf() ? 1.0 / r.w : 0.0;
  return r;
}

// Device-side results of one launch sequence.  The kernels write `rec`; the AC and SSIM kernels
// read `p1g`, the GLOBAL P1 state (single GPU: a copy of rec.p1; slab mode: the rank-ordered
// merge of every slab's state), for mu_e, sigma_e^2 and the global range.
struct DevResults {
  Record rec;
  P1State p1g;
};

// A 3-D field view for the stencil / window kernels: global extents, the planes this launch
// owns (stencil points / window origins), and up to three z-segments of plane storage (in slab
// mode: the lower halo, the local slab and the upper halo received from the neighbour ranks).
// T is the element type of the pair: float (the paper's precision, L330) or double (NEXT f3).
template <typename T>
struct Field3 {
  int64_t nz, ny, nx;        // GLOBAL extents (3-D view, inactive axes squeezed)
  int64_t zown0, zown1;      // owned planes [zown0, zown1)
  int nseg;                  // 1..3
  const T* xs[3];
  const T* ys[3];
  int64_t zs[4];             // segment i holds global planes [zs[i], zs[i+1])
#if defined(__CUDACC__)
  // Plane pointers.  Segment selection uses static indices only (a dynamic index into the
  // by-value kernel parameter would force a local-memory copy of the struct).
  __device__ __forceinline__ const T* xp(int64_t z) const {
    const bool s1 = nseg > 1 && z >= zs[1], s2 = nseg > 2 && z >= zs[2];
    const T* b = s2 ? xs[2] : (s1 ? xs[1] : xs[0]);
    const int64_t z0 = s2 ? zs[2] : (s1 ? zs[1] : zs[0]);
    return b + (z - z0) * (ny * nx);
  }
  __device__ __forceinline__ const T* yp(int64_t z) const {
    const bool s1 = nseg > 1 && z >= zs[1], s2 = nseg > 2 && z >= zs[2];
    const T* b = s2 ? ys[2] : (s1 ? ys[1] : ys[0]);
    const int64_t z0 = s2 ? zs[2] : (s1 ? zs[1] : zs[0]);
    return b + (z - z0) * (ny * nx);
  }
#endif
};

#if defined(__CUDACC__)
// Sequential plane cursor over a Field3 (z increasing by one per step): pointer increments, with
// the segment base re-derived only when a segment boundary is crossed.
template <typename T>
struct PlaneCursor {
  const T* x;
  const T* y;
  int64_t z, next_seg;
  __device__ __forceinline__ void init(const Field3<T>& f, int64_t z0, int64_t off) {
    z = z0;
    x = f.xp(z0) + off;
    y = f.yp(z0) + off;
    next_seg = (f.nseg > 1 && z0 < f.zs[1]) ? f.zs[1] : ((f.nseg > 2 && z0 < f.zs[2]) ? f.zs[2] : INT64_MAX);
  }
  __device__ __forceinline__ void advance(const Field3<T>& f, int64_t off) {
    ++z;
    if (z == next_seg) init(f, z, off);
    else { x += f.ny * f.nx; y += f.ny * f.nx; }
  }
};

// Lighter cursor for hot loops: plane pointers plus the number of planes left in the current
// segment (32-bit); the caller passes the next plane's index only for the rare re-init.
template <typename T>
struct SegCursor {
  const T* x;
  const T* y;
  int left;
  __device__ __forceinline__ void init(const Field3<T>& f, int64_t z0, int64_t off = 0) {
    x = f.xp(z0) + off;
    y = f.yp(z0) + off;
    const int64_t last = f.nseg == 1 ? f.zs[1] : (f.nseg == 2 ? f.zs[2] : f.zs[3]);   // static indices
    const int64_t e = (f.nseg > 1 && z0 < f.zs[1]) ? f.zs[1] : ((f.nseg > 2 && z0 < f.zs[2]) ? f.zs[2] : last);
    left = (int)(e - z0 < INT32_MAX ? e - z0 : INT32_MAX);
  }
  __device__ __forceinline__ void advance(const Field3<T>& f, int64_t znext, int64_t off = 0) {
    if (--left <= 0) init(f, znext, off);
    else { x += f.ny * f.nx; y += f.ny * f.nx; }
  }
  // same with the plane stride (ny * nx) precomputed by the caller
  __device__ __forceinline__ void advance_by(const Field3<T>& f, int64_t znext, int64_t off, int64_t plane) {
    if (--left <= 0) init(f, znext, off);
    else { x += plane; y += plane; }
  }
};

// Element-type helpers: exact min / max in the input type, a (x, y) sample pair.
__device__ __forceinline__ float tmin(float a, float b) { return fminf(a, b); }
__device__ __forceinline__ float tmax(float a, float b) { return fmaxf(a, b); }
__device__ __forceinline__ double tmin(double a, double b) { return fmin(a, b); }
__device__ __forceinline__ double tmax(double a, double b) { return fmax(a, b); }
template <typename T>
struct alignas(2 * sizeof(T)) Pair { T x, y; };
#endif

struct SsimParams {
  int sz, sy, sx;            // steps
  int zchunk;                // origin planes per block
  int range_mode;            // 0 local L, 1 global L
  int64_t nwz, nwy, nwx;     // window-grid extents (debug output indexing)
};

// Ticket counters for the last-block finish (zeroed once; the last block re-arms its counter).
enum : int { TICKET_P1 = 0, TICKET_DERIV = 1, TICKET_SSIM = 2, TICKET_ACZ = 3, TICKET_ACY = 4, TICKET_ACX = 5, TICKET_N = 8 };

#if defined(__CUDACC__)
__device__ __forceinline__ double op_apply(int op, double a, double b) {
  return op == OP_SUM ? a + b : op == OP_MIN ? fmin(a, b) : fmax(a, b);
}
__device__ __forceinline__ double op_identity(int op) {
  return op == OP_SUM ? 0.0 : op == OP_MIN ? dinf() : -dinf();
}

// Returns true in exactly one block: the last to arrive.  All threads of every block call it
// after the block's partial has been written.  Standard threadfence-reduction protocol.
__device__ __forceinline__ bool last_block_arrive(unsigned int* ticket) {
  __shared__ bool s_last;
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0 && threadIdx.y == 0 && threadIdx.z == 0) {
    const unsigned int total = gridDim.x * gridDim.y * gridDim.z;
    const unsigned int t = atomicAdd(ticket, 1u);
    s_last = (t == total - 1);
  }
  __syncthreads();
  if (s_last) __threadfence();
  return s_last;
}

// Block-level combine of a per-thread K-slot record into slot values held by thread 0.
template <int K, typename OpOf>
__device__ void block_reduce_slots(double (&v)[K], OpOf op_of, double* dst_global) {
  __shared__ double s_red[32];
  const int tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  const int nthr = blockDim.x * blockDim.y * blockDim.z;
  const int lane = tid & 31, warp = tid >> 5, nwarps = (nthr + 31) >> 5;
#pragma unroll
  for (int k = 0; k < K; k++) {
    const int op = op_of(k);
    double w = v[k];
    for (int off = 16; off > 0; off >>= 1) w = op_apply(op, w, __shfl_down_sync(0xffffffffu, w, off));
    if (lane == 0) s_red[warp] = w;
    __syncthreads();
    if (warp == 0) {
      double u = lane < nwarps ? s_red[lane] : op_identity(op);
      for (int off = 16; off > 0; off >>= 1) u = op_apply(op, u, __shfl_down_sync(0xffffffffu, u, off));
      if (lane == 0) dst_global[k] = u;
    }
    __syncthreads();
  }
}

// Deterministic combine of K-slot records (run by every thread of the last block, 1-D view of
// the block).  Thread t folds records t, t+T, t+2T, ... in increasing order, all K slots at once
// (K independent loads in flight per record), then the fixed block tree of block_reduce_slots.
// The result depends only on nblocks, never on arrival order.
template <int K, typename OpOf>
__device__ void finish_slots(const double* parts, int nblocks, OpOf op_of, double* out) {
  const int tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  const int nthr = blockDim.x * blockDim.y * blockDim.z;
  double v[K];
#pragma unroll
  for (int k = 0; k < K; k++) v[k] = op_identity(op_of(k));
  for (int b = tid; b < nblocks; b += nthr) {
    const double* p = parts + (size_t)b * K;
#pragma unroll
    for (int k = 0; k < K; k++) v[k] = op_apply(op_of(k), v[k], __ldcg(p + k));
  }
  block_reduce_slots<K>(v, op_of, out);
}


// rcp.approx.ftz.f64 + one Newton step (relative error < 1e-12 for |v| in the float range;
// measured max 8.6e-13, profiles/r01_rcp_probe.txt))
__device__ __forceinline__ double rcp_newton1(double v) {
  double r;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(v));
  return fma(r, fma(-v, r, 1.0), r);
}

// 1/v for finite normal v > 0: rcp.approx (MUFU.RCP64H) + two Newton steps, |rel err| <= 2u.
__device__ __forceinline__ double fast_rcp(double v) {
  double r;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(v));
  double e = fma(-v, r, 1.0);
  r = fma(r, e, r);
  e = fma(-v, r, 1.0);
  return fma(r, e, r);
}

// Opt a kernel into > 48 KB of dynamic shared memory once per device (the attribute persists);
// keeps host API calls out of the per-call launch sequence.
template <auto KERN>
inline cudaError_t set_smem_once(int bytes) {
  static std::atomic<unsigned long long> done{0};
  int dev = 0;
  cudaGetDevice(&dev);
  const unsigned long long bit = 1ull << (dev & 63);
  if (done.load(std::memory_order_acquire) & bit) return cudaSuccess;
  const cudaError_t e = cudaFuncSetAttribute(KERN, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
  if (e == cudaSuccess) done.fetch_or(bit, std::memory_order_release);
  return e;
}

// ---- TMA bulk copies + mbarriers (sm_90+ PTX; UBLKCP / SYNCS in SASS) -------------------------
__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count));
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra WAIT_%=;\n"
      "}\n" ::"r"(smem_addr(bar)), "r"(parity) : "memory");
}
// global -> shared bulk copy (bytes % 16 == 0, both addresses 16-byte aligned), completing on bar
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(smem_addr(dst)), "l"(src), "r"(bytes), "r"(smem_addr(bar)) : "memory");
}

__device__ __forceinline__ float4 ld_stream_f4(const float4* p) {
  float4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  return r;
}

// One 128-bit vector of the input type: 4 floats or 2 doubles, streamed past L1.
template <typename T>
struct Vec16 {
  static constexpr int N = 16 / (int)sizeof(T);
  T e[N];
};
__device__ __forceinline__ Vec16<float> ld_stream16(const float* p) {
  const float4 v = ld_stream_f4(reinterpret_cast<const float4*>(p));
  Vec16<float> r;
  r.e[0] = v.x; r.e[1] = v.y; r.e[2] = v.z; r.e[3] = v.w;
  return r;
}
__device__ __forceinline__ Vec16<double> ld_stream16(const double* p) {
  Vec16<double> r;
  asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0,%1}, [%2];" : "=d"(r.e[0]), "=d"(r.e[1]) : "l"(p));
  return r;
}
#endif

}  // namespace czc

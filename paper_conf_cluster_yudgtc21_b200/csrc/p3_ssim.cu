// p3_ssim.cu — Pattern 3: sliding-window SSIM with a certified fast path.
//
// Paper (L139-L146, Fig. 5, Alg. 3): a w^3 window slides with a fixed step over both
// fields; at each position the window's min, max, sum and power sums are reduced, "mixed (by some
// simple sums and multiplications) to generate the local SSIM", and a global reduction averages
// the local SSIMs.  The paper's kernel keeps per-slice window partials in a shared-memory FIFO of
// depth w along z so each slice is "read and processed only once" (L270, L318), shares the
// x-direction through warp shuffles and the y-direction through shared memory (L270, L320).
//
// B200 design.  A block = 8 warps owns a tile of (32 - WX + 1) x (8 G) window
// origins and a chunk of origin planes, and streams z.  Lane l of warp w owns the footprint
// columns (rows w, w+8, ...; column l) of the tile and, per plane:
//   (a) z-walk — FP64 sums over the last WZ planes of four anchored moments
//         a = x - K,  e = y - x,  a*b (b = y - K),  e*e
//       kept in registers: between resyncs the sums slide (add the entering plane, subtract the
//       leaving one), and every kResync WZ planes they are re-summed from scratch over the
//       window's own planes, so no rounding error lives longer than (kResync + 1) WZ - 1 planes
//       (a large value
//       passing through a running sum would otherwise pollute every later window of the column).
//       The x of the last WZ planes sits in a shifting register ring (the paper's FIFO, moved
//       from window partials to raw samples), which also gives the z-window min/max of x; the
//       y of the leaving plane (and of the ring planes at a resync) is re-read from L2.  The
//       walk also tracks V = max(|a|, |e|) over the planes its sums have touched since the last
//       resync (the error magnitude of the certificate below);
//   (b) y-pass — after ONE __syncthreads on a double-buffered shared-memory exchange of the
//       z-sums, each warp forms running sums over WY rows for its G origin rows;
//   (c) x-pass — power-of-two doubling with warp shuffles across the 32 lanes (the paper's
//       shfl_down x-reduction, L270), then the per-window mix in the cancellation-free form
//         ssim = A/(A + mu_e^2) * B/(B + s_e^2),  A = 2 mu_x mu_y + C1,  B = 2 s_xy + C2
//       (identical to Wang et al.'s formula with C3 = C2/2, reading R14), with L = max - min of
//       the original window (reading R15) or the global range;
//   (d) certificate — an a-posteriori bound on the window's rounding error from V, |K| and the
//       two denominators (derivation at ssim_cert below); a window whose bound exceeds
//       kSsimTau is recomputed exactly (two-pass, anchored at its own first sample) by its warp
//       and counted in czc_result.n_ssim_exact (local anchors + bound +
//       exact fallback).
// K is the block's anchor (tile_anchor: the tile-centre sample of its first plane, or 0 for
// tiles spanning decades or crossing zero), re-chosen at every resync.  Window extents are
// compile-time (cubic 3-D, square 2-D, 1-D).  Round 2: blocks walk long z-chunks where the grid
// is large (launch_t's cost model), and on single-segment float32 fields the footprint planes
// arrive by tensor copies (TMA) into a shared-memory ring instead of per-thread loads.
#include <type_traits>

#include <cuda.h>               // CUtensorMap (encoded through cudaGetDriverEntryPoint)
#include <cudaTypedefs.h>

#include "czc_internal.cuh"

namespace czc {

// Warps per block (A/B, C3 SSIM): 8 (two blocks per SM) 2.94 ms; 12 (one block, 168 registers)
// 3.73 ms; 16 (one block, 128 registers, 1.56 footprint cells per window instead of 1.92) 3.35 ms —
// the per-plane barrier of a single resident block is not hidden by a second one.
#ifndef CZC_P3_WARPS
#define CZC_P3_WARPS 8
#endif
constexpr int kP3Warps = CZC_P3_WARPS;
constexpr int kP3Threads = 32 * kP3Warps;
constexpr double kU = 1.1102230246251565e-16;   // unit roundoff of FP64, 2^-53
// Per-window error budget of the fast path.  The parity tolerance of SSIM is 1e-6 absolute on
// every window and on the mean (north_star); a window whose certified bound exceeds this is
// recomputed exactly.
constexpr double kSsimTau = 2.5e-7;
// The streamed window sums are re-summed from scratch every kResync x (window extent) planes /
// rows and slide in between, so a rounding error lives at most (kResync + 1) w - 1 planes.
// 2: C2 SSIM 0.570 -> 0.554 ms (A/B) against 1, with the same flags on the test fields.
// 3 measured ~1 % faster (C5 169.9 -> 168.1 ms, C3 2.856 -> 2.822 ms) but sends 448 windows of
// the C3 512^3 recipe to the exact path (0 with 2), so 2 stays.
#ifndef CZC_P3_RESYNC
#define CZC_P3_RESYNC 2
#endif
constexpr int kResync = CZC_P3_RESYNC;
#ifndef CZC_P3_LONG_CHUNKS
#define CZC_P3_LONG_CHUNKS 1
#endif
// a new tile anchor at every resync (1) or one per block (0)
#ifndef CZC_P3_REANCHOR
#define CZC_P3_REANCHOR 1
#endif

template <typename T, int WX, int WY, int WZ, int G>
struct SsimGeom {
  static constexpr int TX = 32 - WX + 1;                 // origins per tile along x
  static constexpr int TY = kP3Warps * G;                // origins per tile along y
  static constexpr int FY = TY + WY - 1;                 // footprint rows
  static constexpr int KC = (FY + kP3Warps - 1) / kP3Warps;   // z-walk rows per thread
  static constexpr int ZSTRIDE = FY * 32;                // one component plane of the exchange
  // exchange buffer: { 4 double comps, 2 min/max comps of the input type, 1 float magnitude }
  // x FY x 32, double-buffered
  static constexpr size_t buf_bytes = (size_t)ZSTRIDE * (4 * sizeof(double) + 2 * sizeof(T) + sizeof(float));
  static constexpr size_t smem = 2 * buf_bytes;
  // tensor-copy staging (TMAP): kStages planes of { x, y of the entering plane, y of the plane
  // leaving the z-window }, each a BX x FY float box starting at the 16-byte-aligned column at or
  // before the tile's first column (BX = 36 covers the 32 footprint columns from any offset 0..3)
  static constexpr int BX = 36;
  static constexpr size_t box_bytes = (size_t)BX * FY * sizeof(float);
  static constexpr size_t box_pitch = (box_bytes + 127) / 128 * 128;
  static constexpr size_t ring_off = (smem + 127) / 128 * 128;
  static constexpr int kStages = 3;
  static constexpr size_t smem_tma = ring_off + (size_t)kStages * 3 * box_pitch;
};

__device__ __forceinline__ double shd(double v, int d) { return __shfl_down_sync(0xffffffffu, v, d); }

// Sum over lanes [l, l+W) of v (W compile-time): power-of-two doubling + binary decomposition.
// Lanes whose window leaves the warp return garbage (their origins are outside the tile).
template <int W>
__device__ __forceinline__ double lane_window_sum(double v) {
  double p[5];
  p[0] = v;
#pragma unroll
  for (int k = 1; k < 5; k++)
    if ((1 << k) <= W) p[k] = p[k - 1] + shd(p[k - 1], 1 << (k - 1));
  double r = 0;
  int off = 0;
#pragma unroll
  for (int k = 4; k >= 0; k--) {
    if (W & (1 << k)) {
      r += off == 0 ? p[k] : shd(p[k], off);
      off += 1 << k;
    }
  }
  return r;
}

// min / max over lanes [l, l+W): doubling to the largest power of two <= W, then one
// overlapping combine (max and min are idempotent).
template <int W, bool IS_MAX, typename T>
__device__ __forceinline__ T lane_window_ext(T v) {
  T q = v;
  int k = 0;
#pragma unroll
  for (int j = 1; j < 5; j++)
    if ((1 << j) <= W) {
      const T o = __shfl_down_sync(0xffffffffu, q, 1 << (j - 1));
      q = IS_MAX ? tmax(q, o) : tmin(q, o);
      k = j;
    }
  if ((1 << k) != W) {
    const T o = __shfl_down_sync(0xffffffffu, q, W - (1 << k));
    q = IS_MAX ? tmax(q, o) : tmin(q, o);
  }
  return q;
}

// ---- certificate ---------------------------------------------------------------------------
// Error model of one fast-path window (M samples, anchor K, u = 2^-53).  Every sample i the
// window's sums have touched (the window itself, the <= R WZ - 1 planes before it since the last
// resync, R = kResync, and the <= G - 1 rows above it that the running y-sums add and subtract)
// satisfies
// |a_i|, |e_i| <= V, hence |b_i| <= 2V, |a_i b_i| <= 2V^2, e_i^2 <= V^2.  A sliding sum never
// holds more than W + 1 terms, so with T the term bound of a moment the rounding errors are
//   z-walk: per column <= (WZ - 1) (fresh resync sum) + 2 (R WZ - 1) (slide steps) roundings of
//           partials <= (WZ + 1) T, i.e. <= (1 + 2R) WZ M T over the window's WY WX columns;
//   y-pass: <= (WY - 1) + 2 (G - 1) roundings of partials <= (WY + 1) WZ T per x-column;
//   x-pass: <= 5 doubling levels of partials <= M T;  terms (a, b, e roundings) 3;  1/M: 1;
// so |d Sum| <= cV u M T with cV = (1 + 2R) WZ + WY + 2 G + 13 (incl. slack 4).  With the computed
// means (|true - computed| <= s = 2 cV u V each, incl. their own roundings):
//   |d(S_ab/M)| <= 2 cV u V^2,  |d(S_ee/M)| <= cV u V^2,  |d mu_a|, |d mu_e| <= cV u V,
//   |d s_xy| <= 2 cV u V^2 + (|mu_a| + |mu_b|) 2 cV u V + 8 u V^2        (mu_b = mu_a + mu_e)
//   |d s_ee| <= cV u V^2 + 2 |mu_e| cV u V + 3 u V^2
//   |dB| + |d s_ee| <= (5 cV + 19) u V^2 + cV u V q + u D2,   q = 4 (|mu_a| + |mu_b|) + 2 |mu_e| + 10 s
//   |dA| <= 6 cV u m V + 10 u m^2,  |d mu_e^2| <= 2 cV u V (|mu_e| + s) + (cV u V)^2,
//                                                              m = |mu_x| + |mu_y| + 2 s,
// where D1 = A + mu_e^2 = mu_x^2 + mu_y^2 + C1 and D2 = B + s_ee = s_x^2 + s_y^2 + C2.  Since
// |A| <= D1, mu_e^2 <= 2 D1, |B| <= D2 and s_ee <= 2 D2, each factor of the two-factor form moves
// by at most 2 (|dA| + |d mu_e^2|) / D1 resp. 2 (|dB| + |d s_ee|) / D2, and the mix adds ~10 u:
//   |d ssim| <= n2 / D2 + n1 / D1 + 14 u,
//   n2 = 2 [(5 cV + 19) u V^2 + cV u V q],
//   n1 = 2 [6 cV u m V + 10 u m^2 + 2 cV u V (|mu_e| + s) + (cV u V)^2].
// Evaluated in the cheaper dominating form q' = 8 |mu_a| + 6 |mu_e| + 10 s >= q (|mu_b| <= |mu_a| +
// |mu_e|) and n1' = m (20 u m + 17 cV u V) + 18 (cV u V)^2 >= n1 (the computed |mu_e| <= (|mu_x| +
// |mu_y|)(1 + u) + s since mu_y = mu_x + mu_e is formed from it, and s = 2 cV u V).
// The window is certified when this is <= kSsimTau (cross-multiplied, no division; NaN / inf /
// non-positive denominators fail the test and take the exact path).  Using the computed means
// (not their worst case |K| + 2V) keeps windows near zero (QCLOUD-like fields) certified.
struct SsimCert {
  double cvu, ka, kc, tau;
};
__host__ __device__ constexpr SsimCert ssim_cert(double cV) {
  return SsimCert{cV * kU, 2.0 * kU * (5.0 * cV + 19.0), 20.0 * kU, kSsimTau - 14.0 * kU};
}
// Vf: float magnitude bound (rounded to nearest from the true value: bumped by 2^-22).
__device__ __forceinline__ bool ssim_certified(const SsimCert& c, float Vf, double mua, double mue, double mux,
                                               double muy, double D1, double D2) {
  const double V = (double)Vf * (1.0 + 0x1p-22);
  const double cuV = c.cvu * V;
  const double q = fma(8.0, fabs(mua), fma(6.0, fabs(mue), 20.0 * cuV));        // >= q above
  const double m = fma(4.0, cuV, fabs(mux) + fabs(muy));
  const double n2 = V * fma(c.ka, V, 2.0 * c.cvu * q);
  const double n1 = fma(m, fma(c.kc, m, 17.0 * cuV), 18.0 * cuV * cuV);          // >= n1 above
  return D1 > 0.0 && D2 > 0.0 && fma(n2, D1, n1 * D2) <= c.tau * D1 * D2;
}

// The sample magnitude tracked for the certificate: max(|x - K|, |y - x|), as a float that is
// within one float rounding of the true value (ssim_certified bumps it).
__device__ __forceinline__ float sample_mag(float xs, float ys, float K32, double, double) {
  return fmaxf(fabsf(xs - K32), fabsf(ys - xs));
}
__device__ __forceinline__ float sample_mag(double, double, float, double a, double e) {
  return fmaxf((float)fabs(a), (float)fabs(e));
}

// Butterfly all-reduce over the 32 lanes (every lane gets the same value: IEEE addition, min
// and max are commutative).
__device__ __forceinline__ double warp_allsum(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ double warp_allmin(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmin(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
__device__ __forceinline__ double warp_allmax(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmax(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// Anchor of a tile: the certificate's magnitude V = max |x - K| over the samples a window's sums
// touch, so K should sit near every window's values.  The tile-centre sample does for fields that
// vary little across a tile (temperature-like); for fields spanning decades or crossing zero
// (log-normal densities, QCLOUD-like zeros + clouds) K = 0 keeps |x - K| ~ |x|, which scales with
// the local range L of such fields.  mn / mx: extrema of the tile's first-plane footprint.
template <typename T>
__device__ __forceinline__ T tile_anchor(T centre, T mn, T mx) {
  const bool decades = (mn >= (T)0 && mn < (T)0.25 * mx) || (mx <= (T)0 && mx > (T)0.25 * mn);
  const bool crosses = mn < (T)0 && mx > (T)0;
  return (decades || crosses) ? (T)0 : centre;
}
template <typename T>
__device__ __forceinline__ T warp_min_t(T v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = tmin(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
template <typename T>
__device__ __forceinline__ T warp_max_t(T v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = tmax(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// Exact local SSIM of the window with origin (oz, oy, ox) and extents (wz, wy, wx), computed by
// the whole warp (all lanes must call it with the same arguments; all return the same value):
// the plain definition of L139 / reading R14-R15 — two passes, means about the window's own first
// sample, then centred second moments (no cancellation), FP64 throughout.  The fallback of the
// certified fast path (called only for windows whose bound failed).
template <typename T>
__device__ __forceinline__ double ssim_exact_window(const Field3<T> f, int64_t oz, int64_t oy, int64_t ox, int wz, int wy,
                                                 int wx, bool range_global, double Lglob) {
  const int lane = threadIdx.x & 31;
  const int M = wz * wy * wx;
  const int64_t nx = f.nx;
  const double x0 = (double)f.xp(oz)[oy * nx + ox];
  double sx = 0, sy = 0, mn = x0, mx = x0;
  for (int i = lane; i < M; i += 32) {
    const int ix = i % wx, r = i / wx, iy = r % wy, iz = r / wy;
    const int64_t o = (oy + iy) * nx + ox + ix;
    const double xv = (double)f.xp(oz + iz)[o], yv = (double)f.yp(oz + iz)[o];
    sx += xv - x0;
    sy += yv - x0;
    mn = fmin(mn, xv);
    mx = fmax(mx, xv);
  }
  sx = warp_allsum(sx);
  sy = warp_allsum(sy);
  mn = warp_allmin(mn);
  mx = warp_allmax(mx);
  const double mux = x0 + sx / (double)M, muy = x0 + sy / (double)M;
  double vx = 0, vy = 0, cxy = 0;
  for (int i = lane; i < M; i += 32) {
    const int ix = i % wx, r = i / wx, iy = r % wy, iz = r / wy;
    const int64_t o = (oy + iy) * nx + ox + ix;
    const double dx = (double)f.xp(oz + iz)[o] - mux, dy = (double)f.yp(oz + iz)[o] - muy;
    vx = fma(dx, dx, vx);
    vy = fma(dy, dy, vy);
    cxy = fma(dx, dy, cxy);
  }
  vx = warp_allsum(vx) / (double)M;
  vy = warp_allsum(vy) / (double)M;
  cxy = warp_allsum(cxy) / (double)M;
  double L = range_global ? Lglob : mx - mn;
  L = (L == 0.0) ? 1.0 : L;
  const double C1 = (0.01 * L) * (0.01 * L), C2 = (0.03 * L) * (0.03 * L);
  return ((2.0 * mux * muy + C1) * (2.0 * cxy + C2)) / ((mux * mux + muy * muy + C1) * (vx + vy + C2));
}

// 3-D tensor copy (TMA) of the box at (c0, c1, c2) into shared memory, completing on `bar`;
// elements outside the tensor arrive as zeros
__device__ __forceinline__ void p3_tma_3d(void* dst, const CUtensorMap* map, int c0, int c1, int c2, uint64_t* bar) {
  asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
               :: "r"(smem_addr(dst)), "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(c2), "r"(smem_addr(bar))
               : "memory");
}

// T = float: the x ring and the exchanged extrema are floats (exact); T = double: doubles, one
// block per SM for the larger register ring.
// TMAP (float32 fields; in slab mode the local slab and its upper halo segment): the footprint
// planes arrive by tensor copies issued by one thread kStages - 1 planes ahead into a
// shared-memory ring (no per-thread addresses);
// cells outside the field read zeros (they feed only masked windows, and the tile anchor skips
// them).
template <typename T, int WX, int WY, int WZ, int G, bool TMAP>
__global__ void __launch_bounds__(kP3Threads, (kP3Warps <= 8 && SsimGeom<T, WX, WY, WZ, G>::KC * WZ * sizeof(T) <= 128) ? 2 : 1)
p3_kernel(Field3<T> f, SsimParams p, double* __restrict__ parts, DevResults* __restrict__ res,
          unsigned int* __restrict__ ticket, double* __restrict__ dbg, const __grid_constant__ CUtensorMap mapx,
          const __grid_constant__ CUtensorMap mapy, const __grid_constant__ CUtensorMap mapxh,
          const __grid_constant__ CUtensorMap mapyh, int64_t tz0, int64_t tz1) {
  using Gm = SsimGeom<T, WX, WY, WZ, G>;
  constexpr int TX = Gm::TX, FY = Gm::FY, KC = Gm::KC, ZS = Gm::ZSTRIDE;
  constexpr double invM = 1.0 / (double)(WX * WY * WZ);
  constexpr SsimCert cert = ssim_cert((1.0 + 2.0 * kResync) * WZ + WY + 2.0 * G + 13.0);
  extern __shared__ __align__(128) unsigned char smem_raw[];   // (128: tensor-copy destinations)

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t x0 = (int64_t)blockIdx.x * TX, y0 = (int64_t)blockIdx.y * Gm::TY;
  const int64_t zb = f.zown0 + (int64_t)blockIdx.z * p.zchunk;
  int64_t zo_end = zb + p.zchunk;                         // origin planes [zb, zo_end)
  if (zo_end > f.zown1) zo_end = f.zown1;
  if (zo_end > f.nz - WZ + 1) zo_end = f.nz - WZ + 1;
  const int64_t zend = zo_end > zb ? zo_end + WZ - 1 : zb; // planes [zb, zend)

  int64_t ky = y0 + FY / 2, kx = x0 + 16;
  if (ky > f.ny - 1) ky = f.ny - 1;
  if (kx > f.nx - 1) kx = f.nx - 1;
  const double Lglob = (double)res->p1g.xmax - (double)res->p1g.xmin;

  // In-plane offsets (a plane has < 2^31 elements; the launcher checks).  Footprint rows and
  // columns past the field edge read the clamped edge sample instead of being predicated: they
  // feed only windows whose origin is outside the window grid, which the `ok` mask drops, and
  // every row adds and later subtracts the same samples.
  const int64_t gxc = x0 + lane < f.nx ? x0 + lane : f.nx - 1;
  int off[KC];
#pragma unroll
  for (int k = 0; k < KC; k++) {
    const int64_t gy = y0 + warp + kP3Warps * k;
    off[k] = (int)((gy < f.ny ? gy : f.ny - 1) * f.nx + gxc);
  }
  // Prefetch of plane zb + n (x, y) and of the y sample of the plane leaving the z-window
  // (zb + n - WZ), which is re-read from L2 instead of being kept in the register ring.  Both
  // streams advance through plane cursors (pointer increments, no per-plane address math).
  const int nsteps = (int)(zend - zb);
  SegCursor<T> cin, cold;
  if (nsteps > 0) { cin.init(f, zb); cold.init(f, zb); }
  Pair<T> nxt[KC];                                       // prefetched next plane
  T nyo[KC];                                             // ... and its leaving y sample
  // footprint row warp + kP3Warps k exists (r < FY); warp-uniform, and constant for every k but
  // the last, so rows past the footprint cost nothing
  auto row_live = [&](const int k) { return kP3Warps * (k + 1) <= FY || warp + kP3Warps * k < FY; };
  __shared__ uint64_t s_tbar[Gm::kStages];
  const int xs0 = (int)(x0 & ~(int64_t)3), xsh = (int)(x0 - xs0);   // aligned box column, lane shift
  auto tma_issue = [&](int n) {                          // thread 0; plane n of this block
    if constexpr (TMAP) {
      if (threadIdx.x == 0 && n < nsteps) {
        const int st = n % Gm::kStages;
        const bool old = n >= WZ;
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mbar_expect_tx(&s_tbar[st], (uint32_t)((old ? 3 : 2) * Gm::box_bytes));
        unsigned char* d = smem_raw + Gm::ring_off + (size_t)3 * st * Gm::box_pitch;
        // planes below tz1 come from the segment mapped by (mapx, mapy) (from tz0), the others from
        // the upper halo segment (mapxh, mapyh, from tz1); a leaving plane is always an owned one
        const int64_t z = zb + n;
        const bool hi = z >= tz1;
        const int zc = (int)(hi ? z - tz1 : z - tz0);
        p3_tma_3d(d, hi ? &mapxh : &mapx, xs0, (int)y0, zc, &s_tbar[st]);
        p3_tma_3d(d + Gm::box_pitch, hi ? &mapyh : &mapy, xs0, (int)y0, zc, &s_tbar[st]);
        if (old) p3_tma_3d(d + 2 * Gm::box_pitch, &mapy, xs0, (int)y0, (int)(z - WZ - tz0), &s_tbar[st]);
      }
    }
  };
  auto load = [&](int n, bool has_old) {                 // has_old: n >= WZ (constant per call site)
    if (n < nsteps) {                                    // block-uniform
      if constexpr (TMAP) {
        const int st = n % Gm::kStages;
        mbar_wait(&s_tbar[st], (uint32_t)((n / Gm::kStages) & 1));
        constexpr int BP = (int)(Gm::box_pitch / sizeof(float));
        const float* b = reinterpret_cast<const float*>(smem_raw + Gm::ring_off) + 3 * st * BP;
#pragma unroll
        for (int k = 0; k < KC; k++) {
          if (!row_live(k)) continue;
          const int c = (warp + kP3Warps * k) * Gm::BX + xsh + lane;
          nxt[k].x = b[c];
          nxt[k].y = b[BP + c];
          nyo[k] = has_old ? b[2 * BP + c] : (T)0;
        }
      } else {
#pragma unroll
        for (int k = 0; k < KC; k++) {
          if (!row_live(k)) continue;
          nxt[k].x = __ldg(cin.x + off[k]);
          nxt[k].y = __ldg(cin.y + off[k]);
          nyo[k] = has_old ? __ldg(cold.y + off[k]) : (T)0;
        }
        cin.advance(f, zb + n + 1);
        if (has_old) cold.advance(f, zb + n + 1 - WZ);
      }
    }
  };
  if constexpr (TMAP) {
    if (threadIdx.x == 0) {
#pragma unroll
      for (int i = 0; i < Gm::kStages; i++) mbar_init(&s_tbar[i], 1);
      fence_mbar_init();
    }
    __syncthreads();
#pragma unroll
    for (int n = 0; n + 1 < Gm::kStages; n++) tma_issue(n);
  }

  double sm[KC][4];
  T ring[KC][WZ];                                        // x of the last WZ planes
  float vm[KC];                                          // certificate magnitude of the z-sums
#pragma unroll
  for (int k = 0; k < KC; k++) {
#pragma unroll
    for (int m = 0; m < 4; m++) sm[k][m] = 0;
#pragma unroll
    for (int s = 0; s < WZ; s++) ring[k][s] = 0;
    vm[k] = 0.f;
  }
  load(0, false);
  // The block's anchor (tile_anchor) from the footprint of the plane in `nxt` (one barrier): at
  // the first plane, and again at every resync — the z-sums are re-summed from scratch there, so
  // they can take a new anchor, which keeps K near the values of long z-chunks (a log-normal
  // density changes by decades along z).
  __shared__ T s_ext[2][kP3Warps];
  const bool col_in = x0 + lane < f.nx;
  auto block_anchor = [&](int64_t z) -> T {
    // (TMAP: start from the tile's first sample, which is in the field, and skip the zeros the
    // tensor copies put outside it)
    T mn = TMAP ? f.xp(z)[y0 * f.nx + x0] : nxt[0].x, mx = mn;
#pragma unroll
    for (int k = TMAP ? 0 : 1; k < KC; k++)
      if (row_live(k) && (!TMAP || (col_in && y0 + warp + kP3Warps * k < f.ny))) {
        mn = tmin(mn, nxt[k].x);
        mx = tmax(mx, nxt[k].x);
      }
    mn = warp_min_t(mn);
    mx = warp_max_t(mx);
    if (lane == 0) { s_ext[0][warp] = mn; s_ext[1][warp] = mx; }
    __syncthreads();                                     // (the previous readers passed a barrier)
#pragma unroll
    for (int w = 0; w < kP3Warps; w++) { mn = tmin(mn, s_ext[0][w]); mx = tmax(mx, s_ext[1][w]); }
    return tile_anchor<T>(f.xp(z)[ky * f.nx + kx], mn, mx);
  };
  T Kt = (T)0;
  {
    const T k0 = block_anchor(zb < zend ? zb : f.zown0);
    if (nsteps > 0) Kt = k0;
  }
  double K = (double)Kt;
  float K32 = (float)Kt;

  double ssum = 0;
  unsigned scnt = 0, nexact = 0;
  const bool range_global = p.range_mode != 0;
  // origin-grid membership: x and y are fixed per thread, z advances one plane per step
  const int64_t gxl = x0 + lane;
  const bool xok = lane < TX && gxl <= f.nx - WX && (gxl % p.sx) == 0;
  bool gok[G];
#pragma unroll
  for (int g = 0; g < G; g++) {
    const int64_t gy = y0 + warp * G + g;
    gok[g] = xok && gy <= f.ny - WY && (gy % p.sy) == 0;
  }
  int zph = (int)(zb % p.sz);                            // phase of origin plane zb

  // moments of one sample into s (sign +1: entering, -1: leaving)
  auto add_sample = [&](double (&s)[4], const T xs, const T ys, float& v) {
    const double xd = xs, yd = ys;
    const double a = xd - K, b = yd - K, e = yd - xd;
    s[0] += a; s[1] += e; s[2] = fma(a, b, s[2]); s[3] = fma(e, e, s[3]);
    v = fmaxf(v, sample_mag(xs, ys, K32, a, e));
  };
  auto sub_sample = [&](double (&s)[4], const T xs, const T ys) {
    const double xd = xs, yd = ys;
    const double a = xd - K, b = yd - K, e = yd - xd;
    s[0] -= a; s[1] -= e; s[2] = fma(-a, b, s[2]); s[3] = fma(-e, e, s[3]);
  };

  // One plane step; warm = (step >= WZ: a plane leaves the z-window) and, in the warm-up, s =
  // step are compile-time constants at every call site, so the warm-up planes carry no per-step
  // tests.  resync (block-uniform): re-sum the z-window from scratch instead of sliding.
  auto step_body = [&](const int step, const int s, const bool warm, const bool resync) {
    // the prefetched plane is consumed by the z-walk below, then the next one is requested
    // into the same registers (no copies; its latency hides behind the y / x passes)
    const int buf = step & 1;
    double* Zd = reinterpret_cast<double*>(smem_raw + buf * Gm::buf_bytes);
    T* Zm = reinterpret_cast<T*>(Zd + 4 * ZS);
    float* Zv = reinterpret_cast<float*>(Zm + 2 * ZS);
    const bool full = warm || s == WZ - 1;               // a complete z-window ends here
    // ---- (a) z-walk --------------------------------------------------------------------
    if (resync) {
      // window planes zb+step-WZ+1 .. zb+step: ring slots 1..WZ-1 (x) with their y re-read,
      // plus the entering plane, about a new anchor from the entering plane; V restarts from
      // the window's own samples
#if CZC_P3_REANCHOR
      Kt = block_anchor(zb + step);
      K = (double)Kt;
      K32 = (float)Kt;
#endif
#pragma unroll
      for (int k = 0; k < KC; k++) {
        if (!row_live(k)) continue;
#pragma unroll
        for (int m = 0; m < 4; m++) sm[k][m] = 0;
        vm[k] = 0.f;
      }
#pragma unroll
      for (int t = 1; t < WZ; t++) {
        const T* yr = f.yp(zb + step - WZ + t);
#pragma unroll
        for (int k = 0; k < KC; k++) {
          if (!row_live(k)) continue;
          add_sample(sm[k], ring[k][t], __ldg(yr + off[k]), vm[k]);
        }
      }
    }
#pragma unroll
    for (int k = 0; k < KC; k++) {
      if (!row_live(k)) continue;
      add_sample(sm[k], nxt[k].x, nxt[k].y, vm[k]);
      if (warm && !resync) sub_sample(sm[k], ring[k][0], nyo[k]);
      // shifting ring (oldest plane first; WZ - 1 register moves per row): the main loop is not
      // unrolled, so one copy of the step stays in the instruction cache (the `no_instruction`
      // stalls of an unrolled static-slot ring cost more than the moves: 0.475 -> 0.445 ms)
#pragma unroll
      for (int t = 0; t + 1 < WZ; t++) ring[k][t] = ring[k][t + 1];
      ring[k][WZ - 1] = nxt[k].x;
      const int r = warp + kP3Warps * k;
      if (full) {
        T mn = ring[k][0], mx = ring[k][0];
#pragma unroll
        for (int t = 1; t < WZ; t++) { mn = tmin(mn, ring[k][t]); mx = tmax(mx, ring[k][t]); }
        const int c = r * 32 + lane;
#pragma unroll
        for (int m = 0; m < 4; m++) Zd[m * ZS + c] = sm[k][m];
        Zm[c] = mn;
        Zm[ZS + c] = mx;
        Zv[c] = vm[k];
      }
    }
    load(step + 1, warm || s == WZ - 1);
    if (!full) {                                         // no complete z-window yet
      if constexpr (TMAP) {                              // every thread has read its planes <= step + 1
        __syncthreads();
        tma_issue(step + Gm::kStages - 1);
      }
      return;
    }
    __syncthreads();
    if constexpr (TMAP) tma_issue(step + Gm::kStages - 1);
    const bool zok = zph == 0;                           // origin plane zb + step - WZ + 1
    zph = zph + 1 == p.sz ? 0 : zph + 1;
    // ---- (b) y-pass: the G origin rows of this warp (running sums over WY rows) ------------
    double h[G][4];
    T hmn[G], hmx[G];
    float hv;                                            // V over the union of the G windows' rows
    {
      // y-window min/max: the WY - G + 1 rows shared by all G windows are reduced once
      T cmn = Zm[(warp * G + G - 1) * 32 + lane], cmx = Zm[ZS + (warp * G + G - 1) * 32 + lane];
#pragma unroll
      for (int i = G; i < WY; i++) {
        cmn = tmin(cmn, Zm[(warp * G + i) * 32 + lane]);
        cmx = tmax(cmx, Zm[ZS + (warp * G + i) * 32 + lane]);
      }
      hv = Zv[(warp * G) * 32 + lane];
#pragma unroll
      for (int i = 1; i < G + WY - 1; i++) hv = fmaxf(hv, Zv[(warp * G + i) * 32 + lane]);
#pragma unroll
      for (int g = 0; g < G; g++) {
        const int oy = warp * G + g;
#pragma unroll
        for (int m = 0; m < 4; m++) {
          if (g == 0) {
            double acc = 0;
#pragma unroll
            for (int i = 0; i < WY; i++) acc += Zd[m * ZS + (oy + i) * 32 + lane];
            h[g][m] = acc;
          } else {
            h[g][m] = h[g - 1][m] + (Zd[m * ZS + (oy + WY - 1) * 32 + lane] - Zd[m * ZS + (oy - 1) * 32 + lane]);
          }
        }
        T mn = cmn, mx = cmx;                            // rows [G-1, WY) relative to warp*G
#pragma unroll
        for (int i = g; i < G - 1; i++) {                // rows oy .. warp*G + G - 2
          mn = tmin(mn, Zm[(warp * G + i) * 32 + lane]);
          mx = tmax(mx, Zm[ZS + (warp * G + i) * 32 + lane]);
        }
#pragma unroll
        for (int i = WY; i < WY + g; i++) {              // rows warp*G + WY .. oy + WY - 1
          mn = tmin(mn, Zm[(warp * G + i) * 32 + lane]);
          mx = tmax(mx, Zm[ZS + (warp * G + i) * 32 + lane]);
        }
        hmn[g] = mn;
        hmx[g] = mx;
      }
    }
    // ---- (c) x-pass for all G rows together (independent shuffle chains -> ILP), then mix --
    double S[G][4];
    T wmn[G], wmx[G];
#pragma unroll
    for (int g = 0; g < G; g++) {
#pragma unroll
      for (int m = 0; m < 4; m++) S[g][m] = lane_window_sum<WX>(h[g][m]);
      wmn[g] = lane_window_ext<WX, false>(hmn[g]);
      wmx[g] = lane_window_ext<WX, true>(hmx[g]);
    }
    const float wv = lane_window_ext<WX, true>(hv);
    double ss[G];
    static_assert(G <= 2, "the failed-window mask holds two origin rows");
    unsigned long long fl = 0;                           // bit 32 g + lane: window failed its bound
#pragma unroll
    for (int g = 0; g < G; g++) {
      const bool ok = zok && gok[g];
      // computed by every lane (no divergence); invalid lanes are masked out of the sums
      const double mua = S[g][0] * invM, mue = S[g][1] * invM;
      const double mux = K + mua, muy = mux + mue;
      const double sxy = S[g][2] * invM - mua * (mua + mue);
      const double see = S[g][3] * invM - mue * mue;
      double L = range_global ? Lglob : (double)wmx[g] - (double)wmn[g];
      L = (L == 0.0) ? 1.0 : L;
      const double C1 = (0.01 * L) * (0.01 * L), C2 = (0.03 * L) * (0.03 * L);
      const double A = 2.0 * mux * muy + C1, B = 2.0 * sxy + C2;
      const double D1 = A + mue * mue, D2 = B + see;
      // A, B, D1, D2 > 0 (C1, C2 > 0) up to the certified error; |rel err of the reciprocal| <= 2u
      ss[g] = (A * B) * fast_rcp(D1 * D2);
      // ---- (d) certificate ------------------------------------------------------------------
      const bool flag = ok && !ssim_certified(cert, wv, mua, mue, mux, muy, D1, D2);
      fl |= (unsigned long long)__ballot_sync(0xffffffffu, flag) << (32 * g);
    }
    // failed windows are recomputed exactly by the whole warp (warp-uniform loop, rare)
    while (fl) {
      const int bit = __ffsll((long long)fl) - 1, g = bit >> 5, l = bit & 31;
      fl &= fl - 1;
      const double v = ssim_exact_window<T>(f, zb + step - WZ + 1, y0 + warp * G + g, x0 + l, WZ, WY, WX,
                                            range_global, Lglob);
      if (lane == l) {
#pragma unroll
        for (int q = 0; q < G; q++)
          if (q == g) ss[q] = v;
        nexact++;
      }
    }
#pragma unroll
    for (int g = 0; g < G; g++) {
      const bool ok = zok && gok[g];
      ssum += ok ? ss[g] : 0.0;
      scnt += ok ? 1u : 0u;
      if (dbg && ok) {
        const int64_t oz = zb + step - WZ + 1, gy = y0 + warp * G + g;
        dbg[((oz / p.sz) * p.nwy + gy / p.sy) * p.nwx + (x0 + lane) / p.sx] = ss[g];
      }
    }
  };

  // warm-up: planes 0 .. WZ-1 (the last one completes the first z-window)
#pragma unroll
  for (int s = 0; s < WZ; s++) {
    if (s >= nsteps) break;                              // block-uniform
    step_body(s, s, false, false);
  }
  // steady state: a resync every kResync WZ planes (step = WZ, (1 + kResync) WZ, ...)
  int rph = 0;
#pragma unroll 1
  for (int step = WZ; step < nsteps; step++) {
    step_body(step, 0, true, rph == 0);
    rph = rph + 1 == kResync * WZ ? 0 : rph + 1;
  }

  double rec[kSsimSlots] = {ssum, (double)scnt, (double)nexact};
  const unsigned bid = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
  struct Sum { __device__ int operator()(int) const { return OP_SUM; } };
  __syncthreads();
  block_reduce_slots<kSsimSlots>(rec, Sum{}, parts + (size_t)bid * kSsimSlots);
  if (!last_block_arrive(ticket)) return;
  finish_slots<kSsimSlots>(parts, gridDim.x * gridDim.y * gridDim.z, Sum{}, res->rec.ssim);
  if (tid == 0) *ticket = 0;
}

static inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

// cuTensorMapEncodeTiled through the runtime's driver entry point (no libcuda link): a float32
// plane segment as a (nx, ny, planes) tensor with box (bx, by, 1), zeros outside.
static bool p3_encode_map(CUtensorMap* m, const float* base, int64_t nx, int64_t ny, int64_t nz, int bx, int by) {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    void* fp = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fp, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !fp)
      return false;
    fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fp);
  }
  if (nx % 4 != 0 || ((uintptr_t)base & 15) != 0 || nx >= ((int64_t)1 << 31) || ny >= ((int64_t)1 << 31) ||
      nz >= ((int64_t)1 << 31))
    return false;
  const cuuint64_t dims[3] = {(cuuint64_t)nx, (cuuint64_t)ny, (cuuint64_t)nz};
  const cuuint64_t strides[2] = {(cuuint64_t)nx * 4, (cuuint64_t)(nx * ny) * 4};
  const cuuint32_t box[3] = {(cuuint32_t)bx, (cuuint32_t)by, 1u};
  const cuuint32_t es[3] = {1u, 1u, 1u};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, const_cast<float*>(base), dims, strides, box, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

#ifndef CZC_P3_TMA
#define CZC_P3_TMA 1
#endif

template <typename T, int WX, int WY, int WZ, int G>
static cudaError_t launch_t(const Field3<T>& f, const SsimParams& p, double* parts,
                            DevResults* res, unsigned int* ticket, double* dbg, cudaStream_t st,
                            int64_t* nblocks_out) {
  using Gm = SsimGeom<T, WX, WY, WZ, G>;
  // tensor-copy staging: float32, cubic 3-D windows, one plane segment (single GPU)
  static const CUtensorMap no_map{};
  CUtensorMap mx = no_map, my = no_map, mxh = no_map, myh = no_map;
  int64_t tz0 = 0, tz1 = 0;
  bool tma = false;
  if constexpr (CZC_P3_TMA && std::is_same<T, float>::value && WY > 1 && WZ > 1) {
    // the segment holding the owned planes (the whole field, or the local slab), and the upper
    // halo segment after it when there is one (slab mode: the windows of the last owned planes)
    int seg = -1;
    for (int k = 0; k < f.nseg; k++)
      if (f.zs[k] <= f.zown0 && f.zown1 <= f.zs[k + 1]) seg = k;
    if (seg >= 0 && !nblocks_out) {
      tz0 = f.zs[seg];
      tz1 = f.zs[seg + 1];
      tma = p3_encode_map(&mx, f.xs[seg], f.nx, f.ny, tz1 - tz0, Gm::BX, Gm::FY) &&
            p3_encode_map(&my, f.ys[seg], f.nx, f.ny, tz1 - tz0, Gm::BX, Gm::FY);
      mxh = mx;
      myh = my;
      if (tma && seg + 1 < f.nseg) {
        const int64_t nh = f.zs[seg + 2] - f.zs[seg + 1];
        tma = p3_encode_map(&mxh, f.xs[seg + 1], f.nx, f.ny, nh, Gm::BX, Gm::FY) &&
              p3_encode_map(&myh, f.ys[seg + 1], f.nx, f.ny, nh, Gm::BX, Gm::FY);
      }
    }
  }
  auto kern = tma ? p3_kernel<T, WX, WY, WZ, G, true> : p3_kernel<T, WX, WY, WZ, G, false>;
  const size_t smem_bytes = tma ? Gm::smem_tma : Gm::smem;
  cudaError_t e = tma ? set_smem_once<p3_kernel<T, WX, WY, WZ, G, true>>((int)Gm::smem_tma)
                      : set_smem_once<p3_kernel<T, WX, WY, WZ, G, false>>((int)Gm::smem);
  if (e != cudaSuccess) return e;
  int64_t zhi = f.zown1 < f.nz - WZ + 1 ? f.zown1 : f.nz - WZ + 1;
  const int64_t noz = zhi > f.zown0 ? zhi - f.zown0 : 1;
  const int64_t tiles = cdiv(f.nx - WX + 1, Gm::TX) * cdiv(f.ny - WY + 1, Gm::TY);
  // z-chunking: a block walks zc + WZ - 1 planes for zc window planes; blocks run in waves of
  // `slots` (SMs x resident blocks).  Pick the chunk count that minimises waves x planes per
  // block around the nominal chunk (equal chunks: the longest block walks as few planes as it
  // can), e.g. C2: 3 chunks of 31 instead of 32 + 32 + 29.
  static int occ = 0, sms = 0;
  if (!occ) {
    int d = 0;
    cudaGetDevice(&d);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, d);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, p3_kernel<T, WX, WY, WZ, G, false>, kP3Threads, Gm::smem) !=
            cudaSuccess || occ < 1)
      occ = 1;
  }
  const int64_t slots = (int64_t)(sms > 0 ? sms : 148) * occ;
  const int64_t n0 = cdiv(noz, p.zchunk);
#if CZC_P3_LONG_CHUNKS
  // Any chunk count from the one giving chunks of at most kMaxChunk planes up to n0 + 2: a
  // block's cost is its zc window planes plus its WZ - 1 warm-up planes (z-walk only, ~0.3 of a
  // window plane) plus ~1 plane of prologue / epilogue, times the waves.  Long chunks amortise
  // the warm-up where the grid is large anyway (C3, C5); short ones balance small grids (C2).
#ifndef CZC_P3_MAX_CHUNK
#define CZC_P3_MAX_CHUNK 512
#endif
  constexpr int64_t kMaxChunk = CZC_P3_MAX_CHUNK;
  const int64_t nlo = cdiv(noz, kMaxChunk);
  int64_t best_n = n0, best_cost = INT64_MAX;
  for (int64_t nch = nlo; nch <= n0 + 2 && nch <= noz; nch++) {
    const int64_t zc = cdiv(noz, nch);
    if (cdiv(noz, zc) != nch) continue;               // the same chunking as a smaller count
    const int64_t cost = cdiv(tiles * nch, slots) * (10 * zc + 3 * (WZ - 1) + 10);
    if (cost < best_cost) { best_cost = cost; best_n = nch; }
  }
#else
  int64_t best_n = n0, best_cost = INT64_MAX;
  for (int64_t nch = n0 > 2 ? n0 - 2 : 1; nch <= n0 + 2 && nch <= noz; nch++) {
    const int64_t zc = cdiv(noz, nch);
    if (cdiv(noz, zc) != nch) continue;               // the same chunking as a smaller count
    const int64_t cost = cdiv(tiles * nch, slots) * (zc + WZ - 1);
    if (cost < best_cost) { best_cost = cost; best_n = nch; }
  }
#endif
  SsimParams q = p;
  q.zchunk = (int)cdiv(noz, best_n);
  dim3 grid((unsigned)cdiv(f.nx - WX + 1, Gm::TX), (unsigned)cdiv(f.ny - WY + 1, Gm::TY),
            (unsigned)cdiv(noz, q.zchunk));
  if (nblocks_out) { *nblocks_out = (int64_t)grid.x * grid.y * grid.z; return cudaSuccess; }
  if (f.ny * f.nx >= (int64_t)1 << 31) return cudaErrorInvalidValue;   // 32-bit in-plane offsets
  kern<<<grid, kP3Threads, smem_bytes, st>>>(f, q, parts, res, ticket, dbg, mx, my, mxh, myh, tz0, tz1);
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// 2-D fields (square W x W windows): the rows stream like the planes of the 3-D kernel, and the
// y-window is the running sum of that stream (re-summed from scratch every W rows, as the 3-D
// z-walk), so no shared-memory exchange and no barrier are needed: warp w of a block owns its own
// tile of 32 - W + 1 x-origins (lane = footprint column), keeps FP64 sums of the four anchored
// moments over the last W rows plus the rows' x in a shifting register ring (warm-up peeled),
// re-reads the leaving row's y from L2, and per row does the x-pass by shuffles, the mix and the
// certificate (exact recompute of failed windows by the warp).  (The 3-D kernel on a one-plane
// field ran one plane per block: 0.29 ms for the 1800 x 3600 CESM-shaped pair.)
constexpr int kRowWarps = 8;
template <typename T, int W>
__global__ void __launch_bounds__(kRowWarps * 32)
p3_rows_kernel(Field3<T> f, SsimParams p, int rchunk, double* __restrict__ parts, DevResults* __restrict__ res,
               unsigned int* __restrict__ ticket, double* __restrict__ dbg) {
  constexpr int TX = 32 - W + 1;
  constexpr double invM = 1.0 / (double)(W * W);
  constexpr SsimCert cert = ssim_cert((1.0 + 2.0 * kResync) * W + 1.0 + 2.0 + 13.0);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t ny = f.ny, nx = f.nx;
  const T* __restrict__ X = f.xp(0);
  const T* __restrict__ Y = f.yp(0);
  const int64_t x0 = ((int64_t)blockIdx.x * kRowWarps + warp) * TX;
  const int64_t gx = x0 + lane, gxc = gx < nx ? gx : nx - 1;   // clamped columns feed masked windows only
  const int64_t rb = (int64_t)blockIdx.y * rchunk;
  int64_t ro_end = rb + rchunk;                                 // origin rows [rb, ro_end)
  if (ro_end > ny - W + 1) ro_end = ny - W + 1;
  const int nsteps = ro_end > rb ? (int)(ro_end + W - 1 - rb) : 0;
  const int64_t kx = x0 + 16 < nx ? x0 + 16 : nx - 1, ky = rb + W / 2 < ny ? rb + W / 2 : ny - 1;
  // anchor of this warp's tile (tile_anchor) from its first row
  const T fr = X[rb * nx + gxc];
  T Kt = tile_anchor<T>(X[ky * nx + kx], warp_min_t(fr), warp_max_t(fr));
  double K = (double)Kt;
  float K32 = (float)Kt;
  const double Lglob = res->p1g.xmax - res->p1g.xmin;
  const bool range_global = p.range_mode != 0;
  const bool xok = lane < TX && gx <= nx - W && (gx % p.sx) == 0;
  const T* px = X + rb * nx + gxc;                              // row cursor (next row to load)
  const T* py = Y + rb * nx + gxc;
  const T* pyo = py;                                            // row leaving the window
  T nx_ = 0, ny_ = 0, nyo = 0;
  auto load = [&](int n, bool has_old) {
    if (n < nsteps) {
      nx_ = __ldg(px); ny_ = __ldg(py); px += nx; py += nx;
      if (has_old) { nyo = __ldg(pyo); pyo += nx; }
    }
  };
  double sm[4] = {0, 0, 0, 0};
  float vm = 0.f;
  T ring[W];
#pragma unroll
  for (int t = 0; t < W; t++) ring[t] = 0;
  double ssum = 0;
  unsigned scnt = 0, nexact = 0;
  int rph = (int)(rb % p.sy);
  auto add_sample = [&](const T xs, const T ys) {
    const double xd = xs, yd = ys;
    const double a = xd - K, b = yd - K, e = yd - xd;
    sm[0] += a; sm[1] += e; sm[2] = fma(a, b, sm[2]); sm[3] = fma(e, e, sm[3]);
    vm = fmaxf(vm, sample_mag(xs, ys, K32, a, e));
  };
  load(0, false);
  auto step_body = [&](const int step, const int s, const bool warm, const bool resync) {
    const bool full = warm || s == W - 1;
    if (resync) {                                               // rows rb+step-W+1 .. rb+step
#if CZC_P3_REANCHOR
      // a new anchor from the entering row (the sums restart here), as the 3-D kernel
      Kt = tile_anchor<T>(X[(rb + step) * nx + kx], warp_min_t(nx_), warp_max_t(nx_));
      K = (double)Kt;
      K32 = (float)Kt;
#endif
      sm[0] = sm[1] = sm[2] = sm[3] = 0;
      vm = 0.f;
      const T* yr = Y + (rb + step - W + 1) * nx + gxc;
#pragma unroll
      for (int t = 1; t < W; t++, yr += nx) add_sample(ring[t], __ldg(yr));
    }
    add_sample(nx_, ny_);
    if (warm && !resync) {
      const double xd = ring[0], yd = nyo;
      const double a = xd - K, b = yd - K, e = yd - xd;
      sm[0] -= a; sm[1] -= e; sm[2] = fma(-a, b, sm[2]); sm[3] = fma(-e, e, sm[3]);
    }
#pragma unroll
    for (int t = 0; t + 1 < W; t++) ring[t] = ring[t + 1];     // shifting ring, oldest first
    ring[W - 1] = nx_;
    load(step + 1, warm || s == W - 1);
    if (!full) return;
    T mn = ring[0], mx = ring[0];
#pragma unroll
    for (int t = 1; t < W; t++) { mn = tmin(mn, ring[t]); mx = tmax(mx, ring[t]); }
    const double S0 = lane_window_sum<W>(sm[0]), S1 = lane_window_sum<W>(sm[1]);
    const double S2 = lane_window_sum<W>(sm[2]), S3 = lane_window_sum<W>(sm[3]);
    const T wmn = lane_window_ext<W, false>(mn), wmx = lane_window_ext<W, true>(mx);
    const float wv = lane_window_ext<W, true>(vm);
    const bool ok = xok && rph == 0;                            // origin row rb + step - W + 1
    rph = rph + 1 == p.sy ? 0 : rph + 1;
    const double mua = S0 * invM, mue = S1 * invM;
    const double mux = K + mua, muy = mux + mue;
    const double sxy = S2 * invM - mua * (mua + mue);
    const double see = S3 * invM - mue * mue;
    double L = range_global ? Lglob : (double)wmx - (double)wmn;
    L = (L == 0.0) ? 1.0 : L;
    const double C1 = (0.01 * L) * (0.01 * L), C2 = (0.03 * L) * (0.03 * L);
    const double A = 2.0 * mux * muy + C1, B = 2.0 * sxy + C2;
    const double D1 = A + mue * mue, D2 = B + see;
    double ssim = (A * B) * fast_rcp(D1 * D2);
    const bool flag = ok && !ssim_certified(cert, wv, mua, mue, mux, muy, D1, D2);
    unsigned fl = __ballot_sync(0xffffffffu, flag);
    while (fl) {
      const int l = __ffs(fl) - 1;
      fl &= fl - 1;
      const double v = ssim_exact_window<T>(f, 0, rb + step - W + 1, x0 + l, 1, W, W, range_global, Lglob);
      if (lane == l) { ssim = v; nexact++; }
    }
    ssum += ok ? ssim : 0.0;
    scnt += ok ? 1u : 0u;
    if (dbg && ok) dbg[((rb + step - W + 1) / p.sy) * p.nwx + gx / p.sx] = ssim;
  };
#pragma unroll
  for (int s = 0; s < W; s++) {
    if (s >= nsteps) break;                                     // block-uniform
    step_body(s, s, false, false);
  }
  int qph = 0;
#pragma unroll 1
  for (int step = W; step < nsteps; step++) {
    step_body(step, 0, true, qph == 0);
    qph = qph + 1 == kResync * W ? 0 : qph + 1;
  }
  double rec[kSsimSlots] = {ssum, (double)scnt, (double)nexact};
  struct Sum { __device__ int operator()(int) const { return OP_SUM; } };
  const unsigned bid = blockIdx.x + gridDim.x * blockIdx.y;
  block_reduce_slots<kSsimSlots>(rec, Sum{}, parts + (size_t)bid * kSsimSlots);
  if (!last_block_arrive(ticket)) return;
  finish_slots<kSsimSlots>(parts, gridDim.x * gridDim.y, Sum{}, res->rec.ssim);
  if (threadIdx.x == 0) *ticket = 0;
}

template <typename T, int W>
static cudaError_t launch_rows(const Field3<T>& f, const SsimParams& p, double* parts, DevResults* res,
                               unsigned int* ticket, double* dbg, cudaStream_t st, int64_t* nblocks_out) {
  constexpr int TX = 32 - W + 1;
  const int64_t tiles = cdiv(f.nx - W + 1, TX), bx = cdiv(tiles, kRowWarps);
  const int64_t nro = f.ny - W + 1 > 0 ? f.ny - W + 1 : 1;
  // row chunks: as long as possible (each chunk re-reads W - 1 rows) while the grid still fills
  // about four blocks per SM
  int64_t rc = nro;
  int sms = 148;
  {
    int d = 0;
    cudaGetDevice(&d);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, d);
  }
  while (rc > 4 * W && bx * cdiv(nro, rc) < 4 * (int64_t)sms) rc = cdiv(rc, 2);
  rc = cdiv(nro, cdiv(nro, rc));
  const dim3 grid((unsigned)bx, (unsigned)cdiv(nro, rc), 1);
  if (nblocks_out) { *nblocks_out = (int64_t)grid.x * grid.y; return cudaSuccess; }
  p3_rows_kernel<T, W><<<grid, kRowWarps * 32, 0, st>>>(f, p, (int)rc, parts, res, ticket, dbg);
  return cudaGetLastError();
}

// kind 3: cubic window (3-D); 2: square window, z inactive (2-D); 1: x only (1-D).
template <typename T, int W>
static cudaError_t dispatch_w(int kind, const Field3<T>& f, const SsimParams& p, double* parts,
                              DevResults* res, unsigned int* ticket, double* dbg, cudaStream_t st, int64_t* nb) {
  // keep the z-walk state in registers: float rows of a 2-row origin tile (W <= 8), one origin
  // row per warp otherwise and for double rings (2 blocks per SM instead of 1)
  // (three rows per warp, KC = 4: 492 B of spills at the 128-register cap, C3 SSIM 3.92 ms
  // against 2.85 ms with two, A/B)
  constexpr int G = (W <= 8 && sizeof(T) == 4) ? 2 : 1;
  if (kind == 3) return launch_t<T, W, W, W, G>(f, p, parts, res, ticket, dbg, st, nb);
  if (kind == 2) return launch_rows<T, W>(f, p, parts, res, ticket, dbg, st, nb);
  return launch_t<T, W, 1, 1, 1>(f, p, parts, res, ticket, dbg, st, nb);
}

// Returns cudaErrorInvalidValue for unsupported W.  If nblocks_out != NULL only the grid size
// is computed (no launch).
template <typename T>
cudaError_t launch_ssim(int kind, int W, const Field3<T>& f, const SsimParams& p,
                        double* parts, DevResults* res, unsigned int* ticket, double* dbg,
                        cudaStream_t st, int64_t* nblocks_out) {
  switch (W) {
#define CZC_W(w) case w: return dispatch_w<T, w>(kind, f, p, parts, res, ticket, dbg, st, nblocks_out);
    CZC_W(2) CZC_W(3) CZC_W(4) CZC_W(5) CZC_W(6) CZC_W(7) CZC_W(8) CZC_W(9) CZC_W(10)
    CZC_W(11) CZC_W(12) CZC_W(13) CZC_W(14) CZC_W(15) CZC_W(16)
#undef CZC_W
    default: return cudaErrorInvalidValue;
  }
}
template cudaError_t launch_ssim<float>(int, int, const Field3<float>&, const SsimParams&, double*, DevResults*,
                                        unsigned int*, double*, cudaStream_t, int64_t*);
template cudaError_t launch_ssim<double>(int, int, const Field3<double>&, const SsimParams&, double*, DevResults*,
                                         unsigned int*, double*, cudaStream_t, int64_t*);

}  // namespace czc

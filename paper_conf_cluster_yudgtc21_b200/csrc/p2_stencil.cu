// p2_stencil.cu — Pattern 2: stencil-like metrics.
//
// Paper: Category II (Table I): derivatives, divergence, Laplacian, autocorrelation.
//   Eq. (1): Der(p) = sum_a |f(p+e_a) - f(p-e_a)|   ("a 7-point 3D stencil", L129)
//   L129: divergence / Laplacian are sums of first- / second-order derivatives
//   Alg. 2: central differences (.)/2 and their norm (Grad)
//   Eq. (2): AC(tau) = sum_{p in R_tau} (e_p - mu) (1/3) sum_a (e_{p+tau e_a} - mu) / ne / s^2
// Readings R7, R9, R11, R12, R13.  AC needs P1's mean / variance of the error
// (Alg. 2 takes mu as input, L226): it is read from the device result of P1, no host round trip.
//
// B200 design.
//  * Derivatives: a block owns a 32 x 8 column tile and streams z; the z-neighbours live in
//    registers (prefetched one plane ahead), the in-plane neighbours come from a double-buffered
//    shared-memory plane with a 1-cell halo (one __syncthreads per plane).
//  * Autocorrelation: Eq. 2's sum splits into one lag-product sum per axis,
//      S(tau) = sum_a sum_{p in R_tau} eps_p eps_{p + tau e_a},
//    each computed by a "line walk" along that axis: a thread walks a line, keeps the last TM
//    values of eps in a register ring (static rotation: the walk is unrolled by TM) and adds
//    eps_{i-tau} * eps_i for tau <= min(T, m_line), where m_line is the R_tau bound of the
//    line's other coordinates.  z- and y-walks read coalesced rows directly; the x-walk goes
//    through a warp-private shared-memory transpose.  Every product is formed exactly once.
// FP64 accumulators per thread; block partials combined by the last block in index order.
#include <cuda.h>               // CUtensorMap (the encoder comes through cudaGetDriverEntryPoint)
#include <cudaTypedefs.h>

#include "czc_internal.cuh"

namespace czc {

constexpr int kTX = 32, kTY = 8;
#ifndef CZC_AC_TMA
#define CZC_AC_TMA 1
#endif

// ================================================================================================
// Derivatives
// ================================================================================================
// sqrt for FP64 without the correctly-rounded slow path: rsqrt.approx + two Newton steps,
// relative error ~2^-52 (the oracle's sqrt differs by at most ~1 ulp; metrics are compared with
// a 1e-9 relative tolerance).  sqrt(0) = 0.
__device__ __forceinline__ double fast_sqrt(double a) {
  double r;
  asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(a));
  r = r * fma(-0.5 * a, r * r, 1.5);
  r = r * fma(-0.5 * a, r * r, 1.5);
  const double g = a * r;
  return a > 0.0 ? g : 0.0;
}
__device__ __forceinline__ double dmax(double a, double b) { return a > b ? a : b; }
__device__ __forceinline__ double dmin(double a, double b) { return a < b ? a : b; }

// Derived fields of one point.  ZA / YA: the streamed (slow) axis / the in-plane y axis are
// active; x is always active.  Axis order slow, y, x (slowest first) as in the oracle.  A 2-D
// field is streamed along its rows: its y axis plays the slow axis (ZA, !YA).
// The /2 of the central differences D_a = delta_a / 2 is NOT applied per point: F[GRAD] and
// F[DIV] hold 2 Grad = sqrt(sum delta_a^2) and 2 Div = sum delta_a, and the block's statistics of
// those two fields are scaled once by scale_halved() (power-of-two scaling is exact).  The sums
// start from the first active axis (0 + v is not foldable in IEEE arithmetic: -0).
template <bool ZA, bool YA>
__device__ __forceinline__ void deriv_fields(const double c, const double zp, const double zm,
                                             const double yp, const double ym, const double xp,
                                             const double xm, double F[CZC_NDERIV]) {
  double der1, der2, d2, dsum, lap;
  bool first = true;
  auto axis = [&](const double P, const double M) {
    const double delta = P - M;
    const double l = P - 2.0 * c + M;
    if (first) {
      der1 = fabs(delta); der2 = fabs(l); d2 = delta * delta; dsum = delta; lap = l;
    } else {
      der1 += fabs(delta); der2 += fabs(l); d2 = fma(delta, delta, d2); dsum += delta; lap += l;
    }
    first = false;
  };
  if (ZA) axis(zp, zm);
  if (YA) axis(yp, ym);
  axis(xp, xm);
  F[CZC_DER1] = der1;
  F[CZC_DER2] = der2;
  F[CZC_GRAD] = fast_sqrt(d2);
  F[CZC_DIV] = dsum;
  F[CZC_LAP] = lap;
}

// Undo the factor 2 of F[GRAD] / F[DIV] (deriv_fields) in a block's accumulators:
// max |dF|, sum |dF|, min F, max F scale by 1/2, sum dF^2 by 1/4 — exact.
__device__ __forceinline__ void scale_halved(double (&acc)[kDerivSlots]) {
#pragma unroll
  for (int f : {CZC_GRAD, CZC_DIV}) {
    acc[f * kDerivStats + 0] *= 0.5;
    acc[f * kDerivStats + 1] *= 0.5;
    acc[f * kDerivStats + 2] *= 0.25;
    acc[f * kDerivStats + 3] *= 0.5;
    acc[f * kDerivStats + 4] *= 0.5;
  }
}

// Per-point debug output (czc_config.debug_der): dF = F(y) - F(x) of interior point `idx` (C
// order of the interior grid) for the five fields, field-major with stride nI.  F[GRAD] / F[DIV]
// hold 2 Grad / 2 Div (deriv_fields): their difference is halved, exactly.
__device__ __forceinline__ void deriv_debug(double* dbg, int64_t nI, int64_t idx, const double (&Fx)[CZC_NDERIV],
                                            const double (&Fy)[CZC_NDERIV]) {
#pragma unroll
  for (int f = 0; f < CZC_NDERIV; f++) {
    const double d = Fy[f] - Fx[f];
    dbg[f * nI + idx] = (f == CZC_GRAD || f == CZC_DIV) ? 0.5 * d : d;
  }
}

struct DerivOp {
  __device__ int operator()(int k) const { return deriv_op(k); }
};
struct SumOp {
  __device__ int operator()(int) const { return OP_SUM; }
};

// grid: (ceil(nx/BX), ceil(ny/BY), zchunks); block (BX, BY), BX * BY = 256.
//   3-D fields with nz <= 2: <true, true, 32, 8>; 1-D: <false, false, 256, 1> (3-D fields use
//   deriv3_kernel, 2-D row views deriv2_kernel).
template <typename T, bool ZA, bool YA, int BX, int BY>
__global__ void __launch_bounds__(BX * BY, 2)
deriv_kernel(Field3<T> s, int zchunk, double* __restrict__ parts, DevResults* __restrict__ res,
             unsigned int* __restrict__ ticket, double* __restrict__ dbg) {
  constexpr int kTX = BX, kTY = BY;
  // halo cells of one plane tile: the full ring with a y axis, the two x ends without
  constexpr int kHalo = YA ? 2 * (kTX + 2) + 2 * kTY : 2;
  static_assert(kHalo <= BX * BY, "halo larger than the block");
  __shared__ double2 pl[2][kTY + 2][kTX + 2];     // (x, y) of the current plane, double-buffered
  const int tx = threadIdx.x, ty = threadIdx.y, tid = ty * kTX + tx;
  const int64_t gx = (int64_t)blockIdx.x * kTX + tx, gy = (int64_t)blockIdx.y * kTY + ty;
  constexpr bool az = ZA, ay = YA;
  // interior ranges (reading R11), restricted to the owned planes
  int64_t zlo = az ? 1 : 0, zhi = az ? s.nz - 1 : 1;
  if (zlo < s.zown0) zlo = s.zown0;
  if (zhi > s.zown1) zhi = s.zown1;
  const bool inxy = (ay ? (gy >= 1 && gy < s.ny - 1) : gy == 0) && (gx >= 1 && gx < s.nx - 1);
  const int64_t zb = zlo + (int64_t)blockIdx.z * zchunk;
  int64_t ze = zb + zchunk;
  if (ze > zhi) ze = zhi;

  double acc[kDerivSlots];
#pragma unroll
  for (int k = 0; k < kDerivSlots; k++) acc[k] = op_identity(deriv_op(k));

  const bool own = gx < s.nx && gy < s.ny;
  const int64_t col = own ? gy * s.nx + gx : 0;
  // halo cell of this thread (tid < kHalo): row hr, column hc of the padded tile
  int hr = 0, hc = 0;
  if (!YA) { hr = 1; hc = tid == 0 ? 0 : kTX + 1; }
  else if (tid < 2 * (kTX + 2)) { hr = tid < kTX + 2 ? 0 : kTY + 1; hc = tid % (kTX + 2); }
  else if (tid < kHalo) { const int t = tid - 2 * (kTX + 2); hr = 1 + t % kTY; hc = t < kTY ? 0 : kTX + 1; }
  const int64_t hy = (int64_t)blockIdx.y * kTY + hr - 1, hx = (int64_t)blockIdx.x * kTX + hc - 1;
  const bool hown = tid < kHalo && hy >= 0 && hy < s.ny && hx >= 0 && hx < s.nx;
  const int64_t hcol = hown ? hy * s.nx + hx : 0;

  double xm = 0, x0 = 0, ym = 0, y0 = 0;
  T nxv = 0, nyv = 0, nhx = 0, nhy = 0;               // prefetched: own at z+1, halo at z
  PlaneCursor<T> cown, chalo;                         // own column at z+2, halo cell at z+1
  if (zb < ze) {
    if (own) {
      x0 = s.xp(zb)[col]; y0 = s.yp(zb)[col];
      if (az) {
        xm = s.xp(zb - 1)[col]; ym = s.yp(zb - 1)[col]; nxv = s.xp(zb + 1)[col]; nyv = s.yp(zb + 1)[col];
        if (zb + 2 <= s.nz - 1) cown.init(s, zb + 2, col);
      }
    }
    if (hown) {
      nhx = s.xp(zb)[hcol]; nhy = s.yp(zb)[hcol];
      if (zb + 1 < ze) chalo.init(s, zb + 1, hcol);
    }
  }
  for (int64_t z = zb; z < ze; z++) {
    const int buf = (int)((z - zb) & 1);
    const double xp = az ? (double)nxv : 0.0, yp = az ? (double)nyv : 0.0;
    const T hxv = nhx, hyv = nhy;
    // prefetch: own column at z+2, halo at z+1 (cursors advance one plane per step)
    if (own && az && z + 2 <= s.nz - 1 && z + 1 < ze) { nxv = __ldg(cown.x); nyv = __ldg(cown.y); cown.advance(s, col); }
    if (hown && z + 1 < ze) { nhx = __ldg(chalo.x); nhy = __ldg(chalo.y); chalo.advance(s, hcol); }
    pl[buf][ty + 1][tx + 1] = make_double2(x0, y0);
    if (tid < kHalo) pl[buf][hr][hc] = make_double2(hxv, hyv);
    __syncthreads();
    if (own && inxy) {
      const double2 yn = pl[buf][ty + 2][tx + 1], ys = pl[buf][ty][tx + 1];
      const double2 xe = pl[buf][ty + 1][tx + 2], xw = pl[buf][ty + 1][tx];
      double Fx[CZC_NDERIV], Fy[CZC_NDERIV];
      deriv_fields<ZA, YA>(x0, xp, xm, yn.x, ys.x, xe.x, xw.x, Fx);
      deriv_fields<ZA, YA>(y0, yp, ym, yn.y, ys.y, xe.y, xw.y, Fy);
      if (dbg) {
        const int64_t ix = s.nx - 2, iy = YA ? s.ny - 2 : 1, iz = ZA ? s.nz - 2 : 1;
        deriv_debug(dbg, iz * iy * ix, ((ZA ? z - 1 : 0) * iy + (YA ? gy - 1 : 0)) * ix + gx - 1, Fx, Fy);
      }
#pragma unroll
      for (int fi = 0; fi < CZC_NDERIV; fi++) {
        const double d = Fy[fi] - Fx[fi];
        acc[fi * kDerivStats + 0] = dmax(acc[fi * kDerivStats + 0], fabs(d));
        acc[fi * kDerivStats + 1] += fabs(d);
        acc[fi * kDerivStats + 2] = fma(d, d, acc[fi * kDerivStats + 2]);
        acc[fi * kDerivStats + 3] = dmin(acc[fi * kDerivStats + 3], Fx[fi]);
        acc[fi * kDerivStats + 4] = dmax(acc[fi * kDerivStats + 4], Fx[fi]);
      }
    }
    xm = x0; x0 = xp; ym = y0; y0 = yp;
  }
  __syncthreads();
  scale_halved(acc);
  const unsigned bid = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
  block_reduce_slots<kDerivSlots>(acc, DerivOp{}, parts + (size_t)bid * kDerivSlots);
  if (!last_block_arrive(ticket)) return;
  finish_slots<kDerivSlots>(parts, gridDim.x * gridDim.y * gridDim.z, DerivOp{}, res->rec.deriv);
  if (tid == 0) *ticket = 0;
}

// 2-D fields (row view: the rows stream as the slow axis, ny = 1): lane = column, the row
// neighbours are the previous / next streamed rows in registers, the column neighbours come from
// the adjacent lanes by shuffles (the two warp-edge lanes load their outer neighbour directly),
// so there is no shared-memory plane and no barrier.  One point per thread, 256 columns per block.
template <typename T>
__global__ void __launch_bounds__(256)
deriv2_kernel(Field3<T> s, int zchunk, double* __restrict__ parts, DevResults* __restrict__ res,
              unsigned int* __restrict__ ticket, double* __restrict__ dbg) {
  const int lane = threadIdx.x & 31;
  const int64_t gx = (int64_t)blockIdx.x * 256 + threadIdx.x;
  const int64_t nx = s.nx, nrow = s.nz;
  const int64_t gxc = gx < nx ? gx : nx - 1;
  const bool inx = gx >= 1 && gx < nx - 1;
  int64_t zlo = 1, zhi = nrow - 1;
  if (zlo < s.zown0) zlo = s.zown0;
  if (zhi > s.zown1) zhi = s.zown1;
  const int64_t zb = zlo + (int64_t)blockIdx.z * zchunk;       // grid: (column tiles, 1, row chunks)
  int64_t ze = zb + zchunk;
  if (ze > zhi) ze = zhi;
  double acc[kDerivSlots];
#pragma unroll
  for (int k = 0; k < kDerivSlots; k++) acc[k] = op_identity(deriv_op(k));
  const int n = ze > zb ? (int)(ze - zb) : 0;
  if (n > 0) {
    const T* X = s.xp(0);
    const T* Y = s.yp(0);
    // edge lanes also read the column just outside the warp (clamped inside the row)
    const int64_t ox = lane == 0 ? (gxc > 0 ? gxc - 1 : 0) : (lane == 31 ? (gxc + 1 < nx ? gxc + 1 : nx - 1) : gxc);
    const T* px = X + (zb - 1) * nx;
    const T* py = Y + (zb - 1) * nx;
    double xm = px[gxc], ym = py[gxc];
    px += nx; py += nx;
    double x0 = px[gxc], y0 = py[gxc], xo = px[ox], yo = py[ox];
    px += nx; py += nx;
    T nxv = px[gxc], nyv = py[gxc], nxo = px[ox], nyo = py[ox];   // row zb + 1 (interior rows end at nrow - 2)
    for (int i = 0; i < n; i++) {
      const double xp = nxv, yp = nyv, xpo = nxo, ypo = nyo;
      if (i + 1 < n) {
        px += nx; py += nx;
        nxv = __ldg(px + gxc); nyv = __ldg(py + gxc); nxo = __ldg(px + ox); nyo = __ldg(py + ox);
      }
      // column neighbours of the centre row: lanes +-1, the edge lanes' outer ones from xo / yo
      double xw = __shfl_up_sync(0xffffffffu, x0, 1), yw = __shfl_up_sync(0xffffffffu, y0, 1);
      double xe = __shfl_down_sync(0xffffffffu, x0, 1), ye = __shfl_down_sync(0xffffffffu, y0, 1);
      if (lane == 0) { xw = xo; yw = yo; }
      if (lane == 31) { xe = xo; ye = yo; }
      if (inx) {
        double Fx[CZC_NDERIV], Fy[CZC_NDERIV];
        deriv_fields<true, false>(x0, xp, xm, 0.0, 0.0, xe, xw, Fx);
        deriv_fields<true, false>(y0, yp, ym, 0.0, 0.0, ye, yw, Fy);
        if (dbg) deriv_debug(dbg, (nrow - 2) * (nx - 2), (zb + i - 1) * (nx - 2) + gx - 1, Fx, Fy);
#pragma unroll
        for (int fi = 0; fi < CZC_NDERIV; fi++) {
          const double d = Fy[fi] - Fx[fi];
          acc[fi * kDerivStats + 0] = dmax(acc[fi * kDerivStats + 0], fabs(d));
          acc[fi * kDerivStats + 1] += fabs(d);
          acc[fi * kDerivStats + 2] = fma(d, d, acc[fi * kDerivStats + 2]);
          acc[fi * kDerivStats + 3] = dmin(acc[fi * kDerivStats + 3], Fx[fi]);
          acc[fi * kDerivStats + 4] = dmax(acc[fi * kDerivStats + 4], Fx[fi]);
        }
      }
      xm = x0; ym = y0; x0 = xp; y0 = yp; xo = xpo; yo = ypo;
    }
  }
  scale_halved(acc);
  const unsigned bid = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
  block_reduce_slots<kDerivSlots>(acc, DerivOp{}, parts + (size_t)bid * kDerivSlots);
  if (!last_block_arrive(ticket)) return;
  finish_slots<kDerivSlots>(parts, gridDim.x * gridDim.y * gridDim.z, DerivOp{}, res->rec.deriv);
  if (threadIdx.x == 0) *ticket = 0;
}

// Tile of the 3-D derivative kernel: kDerivTY rows, kDerivPTS points per thread (rows ty, ty + RY,
// ...), kDerivMinB resident blocks per SM (float32; float64: one less).
#ifndef CZC_DERIV_PTS
#define CZC_DERIV_PTS 2
#endif
constexpr int kDerivPTS = CZC_DERIV_PTS;
constexpr int kDerivTY = 4 * kDerivPTS;
template <typename T> constexpr int deriv_minb() { return (kDerivPTS <= 2 ? 4 : 3) - (sizeof(T) == 8 ? 1 : 0); }

// 3-D variant with two points per thread: threads (32, 4) cover a 32 x 8 tile, thread (tx, ty)
// owns rows ty and ty + 4.  The 25 accumulators are shared by both points (half the registers
// per point) and the two independent stencils double each warp's instruction-level parallelism.
template <typename T, int PTS, bool DBG, int TYD, int MINB>
__global__ void __launch_bounds__(kTX * TYD / PTS, MINB)
deriv3_kernel(Field3<T> s, int zc, double* __restrict__ parts, DevResults* __restrict__ res,
              unsigned int* __restrict__ ticket, double* __restrict__ dbg) {
  constexpr int RY = TYD / PTS;                    // thread rows
  constexpr int kHalo = 2 * (kTX + 2) + 2 * TYD;
  static_assert(kHalo <= kTX * RY, "halo larger than the block");
  __shared__ double2 pl[2][TYD + 2][kTX + 2];
  const int tx = threadIdx.x, ty = threadIdx.y, tid = ty * kTX + tx;
  int64_t zlo = 1, zhi = s.nz - 1;
  if (zlo < s.zown0) zlo = s.zown0;
  if (zhi > s.zown1) zhi = s.zown1;
  // Persistent grid (the resident block count), work units = (z-chunk of zc planes, tile) in
  // chunk-major order, dealt round-robin: block b takes units b, b + G, b + 2G, ...  The blocks
  // of one round therefore stream CONSECUTIVE tiles of the same z-chunk in step, so a tile's
  // halo rows / columns (its neighbours' edges) and the chunk's boundary planes are read from
  // DRAM once and from L2 by the neighbour (contiguous tile-major ranges left
  // neighbouring tiles planes apart and read the pair 2.13x per launch).  The chunk count is
  // chosen on the host so the rounds are nearly full.  The accumulators carry across units.
  const int64_t ntxd = (s.nx + kTX - 1) / kTX, ntiles = ntxd * ((s.ny + TYD - 1) / TYD);
  const int64_t planes = zhi > zlo ? zhi - zlo : 0;
  const int64_t nch = planes > 0 ? (planes + zc - 1) / zc : 0, U = ntiles * nch;

  double acc[kDerivSlots];
#pragma unroll
  for (int k = 0; k < kDerivSlots; k++) acc[k] = op_identity(deriv_op(k));
  for (int64_t uu = blockIdx.x; uu < U; uu += gridDim.x) {
  const int64_t chunk = uu / ntiles, tile = uu - chunk * ntiles;
  const int64_t bxi = tile % ntxd, byi = tile / ntxd;
  const int64_t zb = zlo + chunk * zc;
  const int64_t ze = zb + zc < zhi ? zb + zc : zhi;
  const int64_t gx = bxi * kTX + tx, gy0 = byi * TYD + ty;
  __syncthreads();                                   // the previous unit's readers are done with pl

  bool own[PTS], inxy[PTS];
#pragma unroll
  for (int p = 0; p < PTS; p++) {
    const int64_t gy = gy0 + p * RY;
    own[p] = gx < s.nx && gy < s.ny;
    inxy[p] = own[p] && gy >= 1 && gy < s.ny - 1 && gx >= 1 && gx < s.nx - 1;
  }
  const int64_t col = own[0] ? gy0 * s.nx + gx : 0;  // point p: col + p * RY * nx
  const int64_t rstep = (int64_t)RY * s.nx;
  int hr = 0, hc = 0;
  if (tid < 2 * (kTX + 2)) { hr = tid < kTX + 2 ? 0 : TYD + 1; hc = tid % (kTX + 2); }
  else if (tid < kHalo) { const int t = tid - 2 * (kTX + 2); hr = 1 + t % TYD; hc = t < TYD ? 0 : kTX + 1; }
  const int64_t hy = byi * TYD + hr - 1, hx = bxi * kTX + hc - 1;
  const bool hown = tid < kHalo && hy >= 0 && hy < s.ny && hx >= 0 && hx < s.nx;
  const int64_t hcol = hown ? hy * s.nx + hx : 0;

  double xm[PTS], x0[PTS], ym[PTS], y0[PTS];
  T nxv[PTS], nyv[PTS];
  T nhx = 0, nhy = 0;
  SegCursor<T> cown, chalo;                          // own column (row 0) at z+2, halo cell at z+1
  const int64_t plane = s.ny * s.nx;
#pragma unroll
  for (int p = 0; p < PTS; p++) { xm[p] = x0[p] = ym[p] = y0[p] = 0; nxv[p] = nyv[p] = 0; }
  if (zb < ze) {
#pragma unroll
    for (int p = 0; p < PTS; p++) {
      if (own[p]) {
        const int64_t c = col + p * rstep;
        x0[p] = s.xp(zb)[c]; y0[p] = s.yp(zb)[c];
        xm[p] = s.xp(zb - 1)[c]; ym[p] = s.yp(zb - 1)[c];
        nxv[p] = s.xp(zb + 1)[c]; nyv[p] = s.yp(zb + 1)[c];
      }
    }
    if (own[0] && zb + 2 <= s.nz - 1) cown.init(s, zb + 2, col);
    if (hown) {
      nhx = s.xp(zb)[hcol]; nhy = s.yp(zb)[hcol];
      if (zb + 1 < ze) chalo.init(s, zb + 1, hcol);
    }
  }
  // shared-memory slots of this thread (both buffers): centres of its PTS points, its halo cell
  double2* cbase[2];
  double2* hslot[2];
#pragma unroll
  for (int b = 0; b < 2; b++) {
    cbase[b] = &pl[b][ty + 1][tx + 1];
    hslot[b] = &pl[b][hr][hc];
  }
  const int n = ze > zb ? (int)(ze - zb) : 0;
  for (int i = 0; i < n; i++) {
    const int buf = i & 1;
    double xp[PTS], yp[PTS];
#pragma unroll
    for (int p = 0; p < PTS; p++) { xp[p] = (double)nxv[p]; yp[p] = (double)nyv[p]; }
    const T hxv = nhx, hyv = nhy;
    if (i + 1 < n) {
#pragma unroll
      for (int p = 0; p < PTS; p++)
        if (own[p]) { nxv[p] = __ldg(cown.x + p * rstep); nyv[p] = __ldg(cown.y + p * rstep); }
      if (own[0]) cown.advance_by(s, zb + i + 3, col, plane);
      if (hown) { nhx = __ldg(chalo.x); nhy = __ldg(chalo.y); chalo.advance_by(s, zb + i + 2, hcol, plane); }
    }
    double2* cb = buf ? cbase[1] : cbase[0];
#pragma unroll
    for (int p = 0; p < PTS; p++) cb[p * RY * (kTX + 2)] = make_double2(x0[p], y0[p]);
    if (tid < kHalo) *(buf ? hslot[1] : hslot[0]) = make_double2(hxv, hyv);
    __syncthreads();
#pragma unroll
    for (int p = 0; p < PTS; p++) {
      if (inxy[p]) {
        const int r = ty + p * RY + 1;
        const double2 yn = pl[buf][r + 1][tx + 1], ys = pl[buf][r - 1][tx + 1];
        const double2 xe = pl[buf][r][tx + 2], xw = pl[buf][r][tx];
        double Fx[CZC_NDERIV], Fy[CZC_NDERIV];
        deriv_fields<true, true>(x0[p], xp[p], xm[p], yn.x, ys.x, xe.x, xw.x, Fx);
        deriv_fields<true, true>(y0[p], yp[p], ym[p], yn.y, ys.y, xe.y, xw.y, Fy);
        if (DBG)                                   // compile-time: no branch on the timed path
          deriv_debug(dbg, (s.nz - 2) * (s.ny - 2) * (s.nx - 2),
                      ((zb + i - 1) * (s.ny - 2) + gy0 + p * RY - 1) * (s.nx - 2) + gx - 1, Fx, Fy);
#pragma unroll
        for (int fi = 0; fi < CZC_NDERIV; fi++) {
          const double d = Fy[fi] - Fx[fi];
          acc[fi * kDerivStats + 0] = dmax(acc[fi * kDerivStats + 0], fabs(d));
          acc[fi * kDerivStats + 1] += fabs(d);
          acc[fi * kDerivStats + 2] = fma(d, d, acc[fi * kDerivStats + 2]);
          acc[fi * kDerivStats + 3] = dmin(acc[fi * kDerivStats + 3], Fx[fi]);
          acc[fi * kDerivStats + 4] = dmax(acc[fi * kDerivStats + 4], Fx[fi]);
        }
      }
    }
#pragma unroll
    for (int p = 0; p < PTS; p++) { xm[p] = x0[p]; x0[p] = xp[p]; ym[p] = y0[p]; y0[p] = yp[p]; }
  }
  }
  __syncthreads();
  scale_halved(acc);
  const unsigned bid = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
  block_reduce_slots<kDerivSlots>(acc, DerivOp{}, parts + (size_t)bid * kDerivSlots);
  if (!last_block_arrive(ticket)) return;
  finish_slots<kDerivSlots>(parts, gridDim.x * gridDim.y * gridDim.z, DerivOp{}, res->rec.deriv);
  if (tid == 0) *ticket = 0;
}

// ================================================================================================
// Autocorrelation line walks
// ================================================================================================
// One walk step at ring slot S (S is a constant once the caller's loop is unrolled, so the ring
// indexing is static).  The ring holds eps of the last TM positions of the walk, zero-filled for
// positions before the owned range [lo, hi) and for positions >= hi (those points belong to the
// next chunk), so every product eps_{i-t} * eps_i that should not count is exactly 0 * eps_i and
// no per-lag predicate is needed.  The R_tau bound of the line (t <= lim) is applied once, at the
// end (`walk_mask`).
template <int TM>
__device__ __forceinline__ void walk_step(double (&ring)[TM], double (&acc)[TM], double eps, bool keep, int S) {
#pragma unroll
  for (int t = 1; t <= TM; t++) acc[t - 1] = fma(ring[(S - t + 2 * TM) % TM], eps, acc[t - 1]);
  ring[S] = keep ? eps : 0.0;
}

template <int TM>
__device__ __forceinline__ void walk_mask(double (&acc)[TM], int lim) {
#pragma unroll
  for (int t = 1; t <= TM; t++)
    if (t > lim) acc[t - 1] = 0.0;
}

template <int TM>
__device__ __forceinline__ void ac_finish(double (&acc)[TM], double* parts, double* out, unsigned int* ticket) {
  double rec[kAcSlots];
#pragma unroll
  for (int t = 0; t < kAcSlots; t++) rec[t] = 0.0;
#pragma unroll
  for (int t = 0; t < TM; t++) rec[t] = acc[t];
  const unsigned bid = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
  __syncthreads();
  block_reduce_slots<kAcSlots>(rec, SumOp{}, parts + (size_t)bid * kAcSlots);
  if (!last_block_arrive(ticket)) return;
  finish_slots<kAcSlots>(parts, gridDim.x * gridDim.y * gridDim.z, SumOp{}, out);
  if (threadIdx.x + threadIdx.y == 0) *ticket = 0;
}

// Walk of one line.  Positions [lo, end) are visited; points p in [lo, hi) own their products.
// `next` returns the (x, y) sample at the position of a load cursor that runs QD positions
// ahead of the walk: QD loads stay in flight in a register queue whose slot u (of the QD-unrolled
// loop) holds position i0 + u, so both the queue and the ring (QD is a multiple of TM) rotate
// statically.
template <typename T, int TM, int QD, typename Next>
__device__ __forceinline__ void walk_line(Next next, int64_t lo, int64_t hi, int64_t end, double mu,
                                          bool own, double (&ring)[TM], double (&acc)[TM]) {
  static_assert(QD % TM == 0, "queue depth must be a multiple of the ring length");
  T qx[QD], qy[QD];
#pragma unroll
  for (int u = 0; u < QD; u++) {
    qx[u] = 0; qy[u] = 0;
    if (own && lo + u < end) { const Pair<T> v = next(); qx[u] = v.x; qy[u] = v.y; }
  }
  for (int64_t i0 = lo; i0 < end; i0 += QD) {
#pragma unroll
    for (int u = 0; u < QD; u++) {
      const int64_t i = i0 + u;
      if (i < end) {
        const double eps = ((double)qy[u] - (double)qx[u]) - mu;
        if (own && i + QD < end) { const Pair<T> v = next(); qx[u] = v.x; qy[u] = v.y; }
        walk_step<TM>(ring, acc, eps, i < hi, u % TM);
      }
    }
  }
}

// ---- TMA line walks (rows 16-byte aligned: nx % 4 == 0 and aligned segment bases) ------------
// A block's 256 threads own CPT x 256 consecutive x of a row y (thread t: columns t, t + 256, ...)
// and walk positions (planes) i in [lo, end).  Lanes of warp 0 stream the contiguous row segment
// of each position (<= CPT KB per field) into a ring of S = 2 TM shared-memory slots with one bulk
// copy per field, completing on the slot's mbarrier; after every TM positions the block
// synchronises once and the consumed half of the ring is refilled S positions ahead.  Columns past
// the row end read stale slot data; their products are discarded by walk_mask (lim = 0).  CPT = 2
// halves the per-position cost of the waits and barriers per element (float32).
constexpr int kWalkThreads = 256;
template <typename T, int TM, int CPT>
struct BulkWalkSmem {
  static constexpr int S = 2 * TM;
  T x[S][CPT * kWalkThreads];
  T y[S][CPT * kWalkThreads];
  uint64_t bar[S];
};
template <typename T, int TM, int CPT>
__host__ __device__ constexpr int zwalk_tot_offset() { return (int)((sizeof(BulkWalkSmem<T, TM, CPT>) + 15) / 16 * 16); }
template <typename T, int TM, int CPT>
__host__ __device__ constexpr int zwalk_smem() { return zwalk_tot_offset<T, TM, CPT>() + TM * kWalkThreads * (int)sizeof(double); }

// RowPtr(i) -> (const T* xrow, const T* yrow) for position i (already offset to x0).
// Positions are tracked relative to lo in 32 bits.  Lane v < S of warp 0 issues slot v's copies
// (after the barrier that frees the slot), so the refill costs one bulk copy pair per lane.
template <typename T, int TM, int CPT, typename RowPtr>
__device__ __forceinline__ void bulk_walk(BulkWalkSmem<T, TM, CPT>& sm, RowPtr row_ptr, uint32_t bytes, int64_t lo,
                                          int64_t hi, int64_t end, double mu,
                                          double (&ring)[CPT][TM], double (&acc)[CPT][TM], uint32_t& phase) {
  constexpr int S = 2 * TM;
  static_assert(S <= 32, "one phase bit per slot");
  const int tid = threadIdx.x;
  const int jend = (int)(end - lo), jhi = (int)(hi - lo);
  __syncthreads();                                     // barriers initialised; previous line's slots consumed
  auto issue = [&](int slot, int j) {
    const T* xr;
    const T* yr;
    row_ptr(lo + j, xr, yr);
    mbar_expect_tx(&sm.bar[slot], 2 * bytes);
    bulk_g2s(sm.x[slot], xr, bytes, &sm.bar[slot]);
    bulk_g2s(sm.y[slot], yr, bytes, &sm.bar[slot]);
  };
  if (tid < S && tid < jend) issue(tid, tid);
  for (int j0 = 0; j0 < jend; j0 += S) {
#pragma unroll
    for (int u = 0; u < S; u++) {
      const int j = j0 + u;
      if (j < jend) {                                  // block-uniform
        mbar_wait(&sm.bar[u], (phase >> u) & 1u);
        phase ^= 1u << u;
#pragma unroll
        for (int c = 0; c < CPT; c++) {
          const int col = tid + c * kWalkThreads;
          const double eps = ((double)sm.y[u][col] - (double)sm.x[u][col]) - mu;
          walk_step<TM>(ring[c], acc[c], eps, j < jhi, u % TM);
        }
      }
      if (u == TM - 1 || u == S - 1) {                 // half of the ring consumed
        __syncthreads();
        const int v = u - TM + 1 + tid;                // lanes 0..TM-1 refill slots u-TM+1..u
        if (tid < TM && j0 + v + S < jend) issue(v, j0 + v + S);
      }
    }
  }
}

// z-walk, TMA: a line = CPT x 256 consecutive x of row y; persistent grid (the resident block
// count), the (line, owned plane) units in line-major order cut into gridDim.x equal ranges, so
// every block walks ~the same number of planes (a grid of (line, z-chunk) blocks ran 1.7 waves on
// C2) and a range's pieces of two lines each pay their own T halo planes.  The per-line sums are
// masked with the line's R_tau bound and folded into a per-thread total in shared memory.
template <typename E, int TM, int CPT>
__global__ void __launch_bounds__(kWalkThreads, CPT == 1 ? 3 : 2)
ac_zwalk_tma(Field3<E> s, int T, int, double* __restrict__ parts, DevResults* __restrict__ res,
             unsigned int* __restrict__ ticket) {
  extern __shared__ __align__(128) unsigned char walk_smem[];
  using SM = BulkWalkSmem<E, TM, CPT>;
  SM& sm = *reinterpret_cast<SM*>(walk_smem);
  double* tot = reinterpret_cast<double*>(walk_smem + zwalk_tot_offset<E, TM, CPT>());   // [TM][kWalkThreads]
  const int tid = threadIdx.x;
  const double mu = res->p1g.me;
  constexpr int LW = CPT * kWalkThreads;
  const int64_t nzo = s.zown1 - s.zown0, ntx = (s.nx + LW - 1) / LW;
  const int64_t W = ntx * s.ny * nzo;
  const int64_t jb = W * blockIdx.x / gridDim.x, je = W * (blockIdx.x + 1) / gridDim.x;
#pragma unroll
  for (int t = 0; t < TM; t++) tot[t * kWalkThreads + tid] = 0.0;
  if (tid == 0) {
#pragma unroll
    for (int v = 0; v < 2 * TM; v++) mbar_init(&sm.bar[v], 1);
    fence_mbar_init();
  }
  uint32_t phase = 0;
  for (int64_t j = jb; j < je;) {
    const int64_t line = j / nzo, dz = j - line * nzo;
    const int64_t run = (je - j) < (nzo - dz) ? (je - j) : (nzo - dz);
    j += run;
    const int64_t gy = line / ntx, x0 = (line - gy * ntx) * LW;
    int64_t mrow = T;
    if (s.ny > 1 && s.ny - 1 - gy < mrow) mrow = s.ny - 1 - gy;
    const int64_t lo = s.zown0 + dz, hi = lo + run;
    int64_t end = hi + T;
    if (end > s.nz) end = s.nz;
    const int64_t ncols = (s.nx - x0) < LW ? (s.nx - x0) : LW;
    const int64_t off = gy * s.nx + x0;
    double ring[CPT][TM], acc[CPT][TM];
#pragma unroll
    for (int c = 0; c < CPT; c++)
#pragma unroll
      for (int t = 0; t < TM; t++) ring[c][t] = acc[c][t] = 0;
    bulk_walk<E, TM, CPT>(sm, [&](int64_t z, const E*& xr, const E*& yr) { xr = s.xp(z) + off; yr = s.yp(z) + off; },
                          (uint32_t)(ncols * sizeof(E)), lo, hi, end, mu, ring, acc, phase);
    // per column: the R_tau bound from y and x (lim = 0 past the row end), then one sum
#pragma unroll
    for (int c = 0; c < CPT; c++) {
      const int64_t gx = x0 + tid + c * kWalkThreads;
      int64_t m = mrow;
      if (s.nx > 1 && s.nx - 1 - gx < m) m = s.nx - 1 - gx;
      walk_mask<TM>(acc[c], gx < s.nx ? (int)m : 0);
      if (c > 0)
#pragma unroll
        for (int t = 0; t < TM; t++) acc[0][t] += acc[c][t];
    }
#pragma unroll
    for (int t = 0; t < TM; t++) tot[t * kWalkThreads + tid] += acc[0][t];
  }
  double fin[TM];
#pragma unroll
  for (int t = 0; t < TM; t++) fin[t] = tot[t * kWalkThreads + tid];
  ac_finish<TM>(fin, parts, res->rec.ac[0], ticket);
}

// z-walk: thread <-> column (y, x); block 32 x 8 columns; grid.z chunks of owned planes.
template <typename E, int TM>
__global__ void __launch_bounds__(256)
ac_zwalk(Field3<E> s, int T, int zchunk, double* __restrict__ parts, DevResults* __restrict__ res,
         unsigned int* __restrict__ ticket) {
  const int64_t gx = (int64_t)blockIdx.x * kTX + threadIdx.x, gy = (int64_t)blockIdx.y * kTY + threadIdx.y;
  const double mu = res->p1g.me;
  const bool own = gx < s.nx && gy < s.ny;
  int64_t m = T;
  if (s.ny > 1 && s.ny - 1 - gy < m) m = s.ny - 1 - gy;
  if (s.nx > 1 && s.nx - 1 - gx < m) m = s.nx - 1 - gx;
  const int64_t lo = s.zown0 + (int64_t)blockIdx.z * zchunk;
  int64_t hi = lo + zchunk;
  if (hi > s.zown1) hi = s.zown1;
  int64_t end = hi + T;
  if (end > s.nz) end = s.nz;
  const int64_t col = own ? gy * s.nx + gx : 0;
  double ring[TM], acc[TM];
#pragma unroll
  for (int t = 0; t < TM; t++) ring[t] = acc[t] = 0;
  PlaneCursor<E> cur;
  if (own && lo < end) cur.init(s, lo, col);
  walk_line<E, TM, 2 * TM>([&]() {      // read the cursor's plane, then step it (never read past end)
    const Pair<E> v = {__ldg(cur.x), __ldg(cur.y)};
    cur.advance(s, col);
    return v;
  }, lo, hi, end, mu, own, ring, acc);
  walk_mask<TM>(acc, own ? (int)m : 0);
  ac_finish<TM>(acc, parts, res->rec.ac[0], ticket);
}

// x-walk, fast path (rows 16-byte aligned: nx % 4 == 0 and aligned segment bases): lane l of
// each warp owns row (z, y) and streams it with 128-bit loads straight into registers, 4 columns
// per load, two loads in flight ahead; the chunk start lo is a multiple of 4 (xchunk % 4 == 0).
// 32 rows per warp touch 32 lines per load instruction, each line reused over 8 loads (L1).
template <int TM>
__global__ void __launch_bounds__(256)
ac_xwalk_vec(Field3<float> s, int T, int xchunk, double* __restrict__ parts, DevResults* __restrict__ res,
             unsigned int* __restrict__ ticket) {
  constexpr int LCM = (TM % 4 == 0) ? TM : ((TM % 2 == 0) ? 2 * TM : 4 * TM);   // lcm(4, TM)
  constexpr int NV = LCM / 4;                        // float4 vectors per ring period
  const double mu = res->p1g.me;
  const int64_t nrows = (s.zown1 - s.zown0) * s.ny;
  const int64_t myrow = (int64_t)blockIdx.x * 256 + threadIdx.x;
  const bool own = myrow < nrows;
  const int64_t z = own ? s.zown0 + myrow / s.ny : s.zown0, y = own ? myrow % s.ny : 0;
  int64_t m = T;
  if (s.nz > 1 && s.nz - 1 - z < m) m = s.nz - 1 - z;
  if (s.ny > 1 && s.ny - 1 - y < m) m = s.ny - 1 - y;
  const int64_t lo = (int64_t)blockIdx.y * xchunk;
  int64_t hi = lo + xchunk;
  if (hi > s.nx) hi = s.nx;
  int64_t end = hi + T;
  if (end > s.nx) end = s.nx;
  const float4* X = reinterpret_cast<const float4*>(s.xp(z) + y * s.nx + lo);
  const float4* Y = reinterpret_cast<const float4*>(s.yp(z) + y * s.nx + lo);
  const int64_t nvec = (end - lo + 3) / 4;           // the row tail is padded by the next row
  double ring[TM], acc[TM];
#pragma unroll
  for (int t = 0; t < TM; t++) ring[t] = acc[t] = 0;
  float4 ax = make_float4(0, 0, 0, 0), ay = ax, bx = ax, by = ax;
  if (own && nvec > 0) { ax = __ldg(X); ay = __ldg(Y); }
  if (own && nvec > 1) { bx = __ldg(X + 1); by = __ldg(Y + 1); }
  for (int64_t v0 = 0; v0 < nvec; v0 += NV) {
#pragma unroll
    for (int k = 0; k < NV; k++) {
      const int64_t v = v0 + k;
      if (v < nvec) {
        const float4 cx = ax, cy = ay;
        ax = bx; ay = by;
        if (own && v + 2 < nvec) { bx = __ldg(X + v + 2); by = __ldg(Y + v + 2); }
        const float xs4[4] = {cx.x, cx.y, cx.z, cx.w};
        const float ys4[4] = {cy.x, cy.y, cy.z, cy.w};
#pragma unroll
        for (int j = 0; j < 4; j++) {
          const int64_t c = lo + 4 * v + j;
          if (c < end) walk_step<TM>(ring, acc, ((double)ys4[j] - (double)xs4[j]) - mu, c < hi, (4 * k + j) % TM);
        }
      }
    }
  }
  walk_mask<TM>(acc, own ? (int)m : 0);
  ac_finish<TM>(acc, parts, res->rec.ac[2], ticket);
}

// x-walk: each warp owns 32 consecutive rows (z, y); per segment of SEG columns (a multiple of
// TM, so the ring slot of column c is (c - lo) mod TM, static under unrolling) it stages the rows
// coalesced into a warp-private shared-memory tile (transpose), then lane l walks row l.  The
// staged row's (z, y) advance incrementally (no divisions in the loop).
constexpr int kXWarps = 4;   // 4 warps x 32 rows per block (tile: 4 x 32 x <=33 doubles <= 34 KB)
template <typename E, int TM>
__global__ void __launch_bounds__(kXWarps * 32)
ac_xwalk_smem(Field3<E> s, int T, int xchunk, double* __restrict__ parts, DevResults* __restrict__ res,
         unsigned int* __restrict__ ticket) {
  constexpr int SEG = (32 / TM) * TM;
  __shared__ double tile[kXWarps][32][SEG + 1];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const double mu = res->p1g.me;
  const int64_t nrows = (s.zown1 - s.zown0) * s.ny;
  const int64_t row0 = ((int64_t)blockIdx.x * kXWarps + warp) * 32;   // first row of this warp
  const int64_t myrow = row0 + lane;
  const bool own = myrow < nrows;
  const int64_t z = own ? s.zown0 + myrow / s.ny : 0, y = own ? myrow % s.ny : 0;
  int64_t m = T;
  if (s.nz > 1 && s.nz - 1 - z < m) m = s.nz - 1 - z;
  if (s.ny > 1 && s.ny - 1 - y < m) m = s.ny - 1 - y;
  const int64_t lo = (int64_t)blockIdx.y * xchunk;
  int64_t hi = lo + xchunk;
  if (hi > s.nx) hi = s.nx;
  int64_t end = hi + T;
  if (end > s.nx) end = s.nx;
  const int64_t zr0 = s.zown0 + (row0 < nrows ? row0 : 0) / s.ny, yr0 = (row0 < nrows ? row0 : 0) % s.ny;
  double ring[TM], acc[TM];
#pragma unroll
  for (int t = 0; t < TM; t++) ring[t] = acc[t] = 0;
  double (*tl)[SEG + 1] = tile[warp];
  for (int64_t c0 = lo; c0 < end; c0 += SEG) {
    // stage 32 rows x SEG columns of eps, coalesced per row; rows advance (y, z) incrementally
    int64_t zr = zr0, yr = yr0;
    const E* X = s.xp(zr) + yr * s.nx;
    const E* Y = s.yp(zr) + yr * s.nx;
    const int64_t c = c0 + lane;
    const bool cin = lane < SEG && c < end;
#pragma unroll 4
    for (int i = 0; i < 32; i++) {
      double v = 0;
      if (cin && row0 + i < nrows) v = ((double)__ldg(Y + c) - (double)__ldg(X + c)) - mu;
      if (lane < SEG) tl[i][lane] = v;
      if (++yr == s.ny) {
        yr = 0;
        ++zr;
        if (row0 + i + 1 < nrows) { X = s.xp(zr); Y = s.yp(zr); }
      } else {
        X += s.nx;
        Y += s.nx;
      }
    }
    __syncwarp();
    const int64_t ncol = (end - c0) < SEG ? (end - c0) : SEG;
    for (int j0 = 0; j0 < SEG; j0 += TM) {
#pragma unroll
      for (int u = 0; u < TM; u++) {
        const int j = j0 + u;
        if (j < ncol) walk_step<TM>(ring, acc, tl[lane][j], c0 + j < hi, u);
      }
    }
    __syncwarp();
  }
  walk_mask<TM>(acc, own ? (int)m : 0);
  ac_finish<TM>(acc, parts, res->rec.ac[2], ticket);
}

// ---- in-plane lags (x and y) on 2-D tiles ------------------------------------------------------
// For a plane z, the x- and y-lag products of the points of a 64 x 32 tile need eps on the tile
// plus a +TM halo in x and y.  The block stages the raw (x, y) samples of that (32+TM) x (64+TM)
// window with cp.async (16-byte granules when rows are 16-byte aligned, zero-fill outside the
// field), converts them once to eps = (y - x) - mu in a shared double tile (0 outside the field),
// and then every thread walks two short segments with all their values in registers:
//   y-role: column c = tid % 64, rows 8 s .. 8 s + 7 (s = tid / 64): 8 + TM loads, 8 TM FMAs;
//   x-role: row r = tid % 32, columns 8 s .. 8 s + 7 (s = tid / 32): 8 + TM loads, 8 TM FMAs.
// A product eps_p eps_{p + t e_a} belongs to p and counts when p is in Eq. 2's R_t (p + t e_b
// inside the field on every active axis b).  Along the walk axis that holds by the zero fill; the
// other two axes give one bound per thread segment (lim), applied to the segment's lag sums.
// Tiles far from the field ends (all t <= TM valid) skip even that.  The next plane's copies
// overlap the walks of the current one.
// Work split: the (tile, plane) pairs in plane-major order are cut into gridDim.x equal ranges,
// one per block (a persistent grid of the resident block count): no tail wave, and the
// assignment is static, so the result is deterministic.
constexpr int kPlTX = 64, kPlThreads = 256, kPlSeg = 8;
// Tile height: 64 rows where two blocks of the 64 x 64 tile fit an SM (float32, TM <= 10: halo
// 1.34x instead of 1.52x, half the barriers per element), else 32 rows.
template <typename T, int TM> constexpr int pl_ty() { return (sizeof(T) == 4 && TM <= 10) ? 64 : 32; }
template <typename T, int TM> constexpr int pl_bps() { return pl_ty<T, TM>() == 64 ? 2 : (TM <= 10 ? 3 : 2); }
template <typename T, int TM>
struct PlaneTile {
  static_assert(TM % 2 == 0, "even lag templates only");
  static constexpr int TY = pl_ty<T, TM>();
  static constexpr int HX = kPlTX + TM, HY = TY + TM;
  static constexpr int EPG = 16 / (int)sizeof(T);        // elements per 16-byte group
  static constexpr int NV = (HX + EPG - 1) / EPG;        // 16-byte groups per staged row
  static constexpr int PF = EPG * NV;            // staged row pitch (elements), 16-byte multiple
  static constexpr int PE = (PF + 1) | 1;        // eps row pitch (doubles), odd: conflict-free columns
  // staged arrays first, each padded to a multiple of 128 bytes (tensor-copy destinations)
  static constexpr int FPAD = (int)(((HY * PF * sizeof(T) + 127) / 128 * 128 - HY * PF * sizeof(T)) / sizeof(T));
  T fx[HY][PF];
  T padx[FPAD > 0 ? FPAD : 128 / sizeof(T)];
  T fy[HY][PF];
  T pady[FPAD > 0 ? FPAD : 128 / sizeof(T)];
  double e[HY][PE];
};

__device__ __forceinline__ void cp_async4(unsigned dst, const void* src, int src_bytes) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;\n" ::"r"(dst), "l"(src), "r"(src_bytes) : "memory");
}
__device__ __forceinline__ void cp_async8(unsigned dst, const void* src, int src_bytes) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(dst), "l"(src), "r"(src_bytes) : "memory");
}
// one element of the input type, zero-filled when `ok` is false
template <typename T>
__device__ __forceinline__ void cp_async_elem(unsigned dst, const T* src, bool ok) {
  if (sizeof(T) == 4) cp_async4(dst, src, ok ? 4 : 0);
  else cp_async8(dst, src, ok ? 8 : 0);
}
__device__ __forceinline__ void cp_async16(unsigned dst, const void* src, int src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(dst), "l"(src), "r"(src_bytes) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_group 0;\n" ::: "memory"); }

// Stage the window of one plane.  Warp w copies staged rows w, w + 8, ...; VEC: lane l copies the
// 16-byte groups g = l, l + 32, ... of the row (vb = bytes of that group inside the field);
// scalar: lanes copy single samples.  xt / yt point at the tile origin (y0, x0) of the plane.
template <typename T, int TM, bool VEC>
__device__ __forceinline__ void plane_stage(unsigned sfx, const T* xt, const T* yt, int64_t nx, int rv,
                                            int cv, int warp, int lane) {
  using PT = PlaneTile<T, TM>;
  constexpr int HX = PT::HX, HY = PT::HY, NV = PT::NV, PF = PT::PF, EPG = PT::EPG;
  constexpr int RS = kPlThreads / 32;                             // row stride
  constexpr unsigned dy = (unsigned)(offsetof(PT, fy) - offsetof(PT, fx));   // fx -> fy
  if (VEC) {
#pragma unroll
    for (int g = lane; g < NV; g += 32) {
      int vb = cv - EPG * g;
      vb = vb <= 0 ? 0 : (vb >= EPG ? 16 : (int)sizeof(T) * vb);
      const T* px = xt + warp * nx + EPG * g;
      const T* py = yt + warp * nx + EPG * g;
      unsigned d = sfx + (unsigned)(sizeof(T) * (warp * PF + EPG * g));
      for (int r = warp; r < HY; r += RS) {
        if (r < rv) {
          cp_async16(d, px, vb);
          cp_async16(d + dy, py, vb);
        } else {                                                  // below the field: zero fill
          cp_async16(d, xt, 0);
          cp_async16(d + dy, yt, 0);
        }
        px += RS * nx; py += RS * nx; d += sizeof(T) * RS * PF;
      }
    }
  } else {
    for (int r = warp; r < HY; r += RS) {
#pragma unroll
      for (int c0 = 0; c0 < HX; c0 += 32) {
        const int c = c0 + lane;
        if (c < HX) {
          const bool ok = r < rv && c < cv;
          const int64_t o = ok ? r * nx + c : 0;
          const unsigned d = sfx + (unsigned)(sizeof(T) * (r * PF + c));
          cp_async_elem(d, xt + o, ok);
          cp_async_elem(d + dy, yt + o, ok);
        }
      }
    }
  }
  cp_async_commit();
}

// Lag products of one segment v[0 .. 8 + TM): points j < 8 own v[j] * v[j + t].  With LIM, the
// segment's lag-t sum counts only if t <= lim.
template <int TM, bool LIM>
__device__ __forceinline__ void seg_products(const double (&v)[kPlSeg + TM], int lim, double (&acc)[TM]) {
#pragma unroll
  for (int t = 1; t <= TM; t++) {
    if (!LIM) {
#pragma unroll
      for (int j = 0; j < kPlSeg; j++) acc[t - 1] = fma(v[j], v[j + t], acc[t - 1]);
    } else {
      double part = 0.0;
#pragma unroll
      for (int j = 0; j < kPlSeg; j++) part = fma(v[j], v[j + t], part);
      acc[t - 1] += t <= lim ? part : 0.0;
    }
  }
}

// limx: R_t bound of the y-role's column (from x), limy: of the x-role's row (from y), both
// already capped by the plane's z bound.
template <typename T, int TM, bool LIM>
__device__ __forceinline__ void plane_walks(const PlaneTile<T, TM>& sm, int tid, int limx, const int (&limy)[PlaneTile<T, TM>::TY / 32],
                                            double (&acc)[TM]) {
  constexpr int NH = PlaneTile<T, TM>::TY / 32;     // 32-row halves of the tile
  static_assert(NH == 1 || NH == 2, "tile heights 32 and 64");
  double v[kPlSeg + TM];
#pragma unroll 1
  for (int h = 0; h < NH; h++) {
    {  // y-role
      const int c = tid & (kPlTX - 1), ys = (tid / kPlTX) * kPlSeg + 32 * h;
#pragma unroll
      for (int j = 0; j < kPlSeg + TM; j++) v[j] = sm.e[ys + j][c];
      seg_products<TM, LIM>(v, limx, acc);
    }
    {  // x-role
      const int r = (tid & 31) + 32 * h, xs = (tid / 32) * kPlSeg;
#pragma unroll
      for (int j = 0; j < kPlSeg + TM; j++) v[j] = sm.e[r][xs + j];
      seg_products<TM, LIM>(v, h == 0 ? limy[0] : limy[NH - 1], acc);   // NH <= 2: no local array
    }
  }
}

// grid: persistent (gridDim.x blocks); block 256; requires ny > 1.
// VEC: rows 16-byte aligned (nx % 4 == 0, aligned plane segments) and (32 + TM) * nx < 2^31.
// One 3-D tensor copy (TMA, cp.async.bulk.tensor) of the box at (c0, c1, c2) into shared memory,
// completing on `bar`; elements outside the tensor arrive as zeros.
__device__ __forceinline__ void tma_load_3d(void* dst, const CUtensorMap* map, int c0, int c1, int c2, uint64_t* bar) {
  asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
               :: "r"(smem_addr(dst)), "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(c2), "r"(smem_addr(bar))
               : "memory");
}

// TMAP (float32, one plane segment): the x / y windows arrive by two tensor copies issued by one
// thread (mapx / mapy: the segment as a (nx, ny, planes) tensor, box (PF, HY, 1)) instead of
// per-thread 16-byte cp.async groups.
template <typename T, int TM, bool VEC, bool TMAP>
__global__ void __launch_bounds__(kPlThreads, pl_bps<T, TM>())
ac_plane(Field3<T> s, double* __restrict__ parts, DevResults* __restrict__ res, unsigned int* __restrict__ ticket,
         const __grid_constant__ CUtensorMap mapx, const __grid_constant__ CUtensorMap mapy, int64_t map_z0) {
  extern __shared__ __align__(128) unsigned char plane_smem[];
  using PT = PlaneTile<T, TM>;
  PT& sm = *reinterpret_cast<PT*>(plane_smem);
  static_assert(!TMAP || (sizeof(T) == 4 && offsetof(PT, fy) % 128 == 0), "tensor copies: float32, 128-byte aligned");
  __shared__ uint64_t s_bar;
  uint32_t phase = 0;
  if constexpr (TMAP) {
    if (threadIdx.x == 0) { mbar_init(&s_bar, 1); fence_mbar_init(); }
    __syncthreads();
  }
  constexpr int HY = PT::HY, NV = PT::NV, EPG = PT::EPG;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const unsigned sfx = (unsigned)__cvta_generic_to_shared(&sm.fx[0][0]);
  const int r0 = tid / NV, g0 = tid % NV;          // this thread's first conversion group
  const double mu = res->p1g.me;
  const int64_t nzo = s.zown1 - s.zown0, ntx = (s.nx + kPlTX - 1) / kPlTX;
  constexpr int TY = PT::TY, NH = TY / 32;
  const int64_t ntiles = ntx * ((s.ny + TY - 1) / TY), W = ntiles * nzo;
  const int64_t jb = W * blockIdx.x / gridDim.x, je = W * (blockIdx.x + 1) / gridDim.x;
  double acc[TM];
#pragma unroll
  for (int t = 0; t < TM; t++) acc[t] = 0;
  // Items (plane, tile) in plane-major order, x-tiles fastest: the blocks sweep the field a few
  // planes apart, so a tile's +TM halo (its x / y neighbours' cells) is read from DRAM once and
  // from L2 by the neighbour's block (tile-major z-runs left the blocks planes apart and the
  // halo re-read from DRAM: 352 MB per launch on C2 for a 200 MB pair).
  // The item origin advances incrementally (one 64-bit division per block, not per item).
  int64_t z, x0, y0;
  {
    const int64_t q = jb / ntiles, tile = jb - q * ntiles;
    z = s.zown0 + q;
    x0 = (tile % ntx) * kPlTX;
    y0 = (tile / ntx) * TY;
  }
  auto next_org = [&](int64_t& nz, int64_t& nx0, int64_t& ny0) {
    nx0 += kPlTX;
    if (nx0 >= s.nx) {
      nx0 = 0;
      ny0 += TY;
      if (ny0 >= s.ny) { ny0 = 0; ++nz; }
    }
  };
  auto stage_item = [&](int64_t sz, int64_t sx0, int64_t sy0) {
    const int rv = (int)(s.ny - sy0 < HY ? s.ny - sy0 : HY);
    const int cv = (int)(s.nx - sx0 < PT::PF ? s.nx - sx0 : PT::PF);
    if constexpr (TMAP) {
      (void)rv; (void)cv;
      if (threadIdx.x == 0) {
        // the previous readers of the staging buffers passed a barrier; order their generic-proxy
        // reads before the async-proxy writes
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mbar_expect_tx(&s_bar, (uint32_t)(2 * HY * PT::PF * sizeof(T)));
        const int zc = (int)(sz - map_z0);               // plane within the mapped segment
        tma_load_3d(&sm.fx[0][0], &mapx, (int)sx0, (int)sy0, zc, &s_bar);
        tma_load_3d(&sm.fy[0][0], &mapy, (int)sx0, (int)sy0, zc, &s_bar);
      }
    } else {
      const int64_t o = sy0 * s.nx + sx0;
      plane_stage<T, TM, VEC>(sfx, s.xp(sz) + o, s.yp(sz) + o, s.nx, rv, cv, warp, lane);
    }
  };
  if (jb < je) stage_item(z, x0, y0);
  for (int64_t j = jb; j < je; j++) {
    const bool xy_inner = x0 + kPlTX + TM <= s.nx && y0 + TY + TM <= s.ny;
    // staged cells outside the field hold eps = 0
    const int rv = (int)(s.ny - y0 < HY ? s.ny - y0 : HY);
    const int cv = (int)(s.nx - x0 < PT::PF ? s.nx - x0 : PT::PF);
    // per-segment R_t bounds from x (y-role column) and y (x-role row)
    const int64_t mx = s.nx - 1 - (x0 + (tid & (kPlTX - 1)));
    const int limx0 = mx < TM ? (int)(mx < -1 ? -1 : mx) : TM;
    int limy0[NH];
#pragma unroll
    for (int h = 0; h < NH; h++) {
      const int64_t my = s.ny - 1 - (y0 + (tid & 31) + 32 * h);
      limy0[h] = my < TM ? (int)(my < -1 ? -1 : my) : TM;
    }
    {
      if constexpr (TMAP) {
        mbar_wait(&s_bar, phase);
        phase ^= 1u;
      } else {
        cp_async_wait_all();
      }
      __syncthreads();                     // plane z staged; previous walks done with sm.e
      {
        // all 16-byte groups of the staged window, 256 at a time (row r, group g of the row);
        // tiles away from the field ends (xy_inner, block-uniform) need no zero fill
        auto convert = [&](const bool inner) {
          int r = r0, g = g0;
          for (int i = tid; i < HY * NV; i += kPlThreads) {
            const Vec16<T> a = *reinterpret_cast<const Vec16<T>*>(&sm.fx[r][EPG * g]);
            const Vec16<T> b = *reinterpret_cast<const Vec16<T>*>(&sm.fy[r][EPG * g]);
            double* er = &sm.e[r][EPG * g];
#pragma unroll
            for (int j = 0; j < EPG; j++) {
              const double ej = ((double)b.e[j] - (double)a.e[j]) - mu;
              er[j] = (inner || (r < rv && EPG * g + j < cv)) ? ej : 0.0;
            }
            r += kPlThreads / NV;
            g += kPlThreads % NV;
            if (g >= NV) { g -= NV; r++; }
          }
        };
        if (xy_inner) convert(true);
        else convert(false);
      }
      __syncthreads();                     // eps ready, staging buffer free
      int64_t nz = z, nx0 = x0, ny0 = y0;
      next_org(nz, nx0, ny0);
      if (j + 1 < je) stage_item(nz, nx0, ny0);
      // R_t bound from the z axis (active only for 3-D fields)
      const int64_t mz64 = s.nz > 1 ? s.nz - 1 - z : TM;
      const int mz = mz64 > TM ? TM : (int)mz64;
      if (xy_inner && mz >= TM) {
        int full[NH];
#pragma unroll
        for (int h = 0; h < NH; h++) full[h] = TM;
        plane_walks<T, TM, false>(sm, tid, TM, full, acc);
      } else {
        int ly[NH];
#pragma unroll
        for (int h = 0; h < NH; h++) ly[h] = limy0[h] < mz ? limy0[h] : mz;
        plane_walks<T, TM, true>(sm, tid, limx0 < mz ? limx0 : mz, ly, acc);
      }
      z = nz; x0 = nx0; y0 = ny0;
    }
  }
  ac_finish<TM>(acc, parts, res->rec.ac[1], ticket);
}

// cuTensorMapEncodeTiled through the runtime's driver entry point (no libcuda link): a float32
// segment of planes as a (nx, ny, planes) tensor with box (bx, by, 1), zeros outside.
static bool encode_plane_map(CUtensorMap* m, const float* base, int64_t nx, int64_t ny, int64_t nz, int bx, int by) {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    void* fp = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fp, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !fp)
      return false;
    fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fp);
  }
  if (nx % 4 != 0 || ((uintptr_t)base & 15) != 0 || nx >= ((int64_t)1 << 32) || ny >= ((int64_t)1 << 32) ||
      nz >= ((int64_t)1 << 32))
    return false;
  const cuuint64_t dims[3] = {(cuuint64_t)nx, (cuuint64_t)ny, (cuuint64_t)nz};
  const cuuint64_t strides[2] = {(cuuint64_t)nx * 4, (cuuint64_t)(nx * ny) * 4};
  const cuuint32_t box[3] = {(cuuint32_t)bx, (cuuint32_t)by, 1u};
  const cuuint32_t es[3] = {1u, 1u, 1u};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, const_cast<float*>(base), dims, strides, box, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}
static bool encode_plane_map(CUtensorMap*, const double*, int64_t, int64_t, int64_t, int, int) { return false; }

static inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }
static int sm_count() {
  int d = 0, n = 0;
  cudaGetDevice(&d);
  cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, d);
  return n > 0 ? n : 1;
}

template <typename T>
static int64_t deriv_zplanes(const Field3<T>& s) {
  int64_t zlo = s.nz > 1 ? 1 : 0, zhi = s.nz > 1 ? s.nz - 1 : 1;
  if (zlo < s.zown0) zlo = s.zown0;
  if (zhi > s.zown1) zhi = s.zown1;
  return zhi > zlo ? zhi - zlo : 1;
}
// 2-D fields (one plane, never slab-sharded) are streamed along their rows: view (ny, 1, nx).
template <typename T>
static Field3<T> deriv_view(const Field3<T>& s) {
  if (!(s.nz == 1 && s.ny > 1)) return s;
  Field3<T> v = s;
  v.nz = s.ny; v.ny = 1;
  v.zown0 = 0; v.zown1 = s.ny;
  v.zs[0] = 0; v.zs[1] = s.ny;
  return v;
}
// Launch shape: (BX, BY) tiles x chunks of the streamed axis; the chunk length is the requested
// one unless that leaves fewer than ~4 blocks per SM (short or 2-D fields), never below 8 planes
// (4 rather than 8: C2 runs one 98-plane chunk per tile, derivatives 0.307 -> 0.290 ms).
template <typename T>
static dim3 deriv_grid(const Field3<T>& s, int zchunk, int* zc) {
  const int bx = s.ny > 1 ? kTX : 256, by = s.ny > 1 ? (s.nz > 2 ? kDerivTY : kTY) : 1;
  const int64_t tiles = cdiv(s.nx, bx) * cdiv(s.ny, by), planes = deriv_zplanes(s);
  if (s.ny > 1 && s.nz > 2) {                 // deriv3_kernel: persistent, resident block count
    // z-chunks: the count whose round-robin rounds are fullest; a unit costs its planes plus ~1
    // plane's worth of start-up (three planes loaded before the first point, no prefetch across
    // units: on C2, 12 units of 14 planes per block ran 0.281 ms against 0.268 ms for the old
    // contiguous split, 167 planes in ~2 pieces, at 2.1x the DRAM traffic); at most planes / 8
    // chunks
    const int64_t G = (int64_t)sm_count() * deriv_minb<T>();
    int64_t best = 1;
    double best_cost = 1e300;
    for (int64_t nch = 1; nch <= (planes / 8 > 1 ? planes / 8 : 1); nch++) {
      const int64_t zc_ = cdiv(planes, nch), U = tiles * cdiv(planes, zc_);
      const double rounds = (double)cdiv(U, G);
      const double cost = rounds * (double)(zc_ + 1);     // planes a block walks (critical path)
      if (cost < best_cost * 0.999) { best_cost = cost; best = nch; }
    }
    *zc = (int)cdiv(planes, best);
    const int64_t U = tiles * cdiv(planes, *zc);
    return dim3((unsigned)(U < G ? (U > 0 ? U : 1) : G), 1, 1);
  }
  int64_t c = zchunk;
  const int64_t fill = cdiv(planes * tiles, (int64_t)sm_count() * 4);
  if (fill < c) c = fill < 8 ? 8 : fill;
  c = cdiv(planes, cdiv(planes, c));          // equal chunks
  *zc = (int)c;
  return dim3((unsigned)cdiv(s.nx, bx), (unsigned)cdiv(s.ny, by), (unsigned)cdiv(planes, c));
}
template <typename T>
int64_t deriv_blocks(const Field3<T>& s0, int zchunk) {
  int zc;
  const dim3 g = deriv_grid(deriv_view(s0), zchunk, &zc);
  return (int64_t)g.x * g.y * g.z;
}

template <typename T>
cudaError_t launch_deriv(const Field3<T>& s0, int zchunk, double* parts, DevResults* res,
                         unsigned int* ticket, double* dbg, cudaStream_t st) {
  const Field3<T> s = deriv_view(s0);
  int zc;
  const dim3 grid = deriv_grid(s, zchunk, &zc);
  if (s.ny > 1 && s.nz > 2) {
    const dim3 blk(kTX, kDerivTY / kDerivPTS);
    if (dbg) deriv3_kernel<T, kDerivPTS, true, kDerivTY, deriv_minb<T>()><<<grid, blk, 0, st>>>(s, zc, parts, res, ticket, dbg);
    else deriv3_kernel<T, kDerivPTS, false, kDerivTY, deriv_minb<T>()><<<grid, blk, 0, st>>>(s, zc, parts, res, ticket, dbg);
  }
  else if (s.ny > 1) deriv_kernel<T, true, true, kTX, kTY><<<grid, dim3(kTX, kTY), 0, st>>>(s, zc, parts, res, ticket, dbg);
  else if (s.nz > 1) deriv2_kernel<T><<<grid, 256, 0, st>>>(s, zc, parts, res, ticket, dbg);
  else deriv_kernel<T, false, false, 256, 1><<<grid, dim3(256, 1), 0, st>>>(s, zc, parts, res, ticket, dbg);
  return cudaGetLastError();
}

// Autocorrelation: the z-walk (3-D fields) and the in-plane tile kernel (x and y lags, ny > 1),
// or the x-walk alone for 1-D fields; each launch has its own partial-buffer slice and ticket and
// writes its own record slot (z -> ac[0], in-plane -> ac[1], x-walk -> ac[2]); the finish sums them.
// columns per thread of the TMA z-walk: 2 for float32 (2 KB row segments), 1 for float64
template <typename E>
constexpr int kWalkCPT = sizeof(E) == 4 ? 2 : 1;

struct AcGrids {
  dim3 z, zt, pl, x, xvec;
  bool rz, ry, rx;
  int zc, pzc, xc;
};
template <typename E>
static AcGrids ac_grids(const Field3<E>& s, int T) {
  AcGrids g{};
  const int64_t nzo = s.zown1 - s.zown0;
  g.xc = 128;                // xc % 4 == 0 for the vector x-walk
  // z-walk chunks: long walks amortise the T halo planes every chunk re-reads (measured: 50 ->
  // 100 -> 256 planes made the C3 walk 0.99 -> 0.91 -> 0.86 ms, and C2's 100 planes in one chunk
  // beat two chunks of 50: 0.209 vs 0.226 ms); shorter only when the grid would not fill the 2
  // resident blocks per SM once; equal chunks
  {
    const int64_t xy = cdiv(s.nx, kWalkCPT<E> * kWalkThreads) * s.ny;
    int64_t zc = 256;
    while (zc > 16 && xy * cdiv(nzo, zc) < 2 * (int64_t)sm_count()) zc /= 2;
    zc = cdiv(nzo, cdiv(nzo, zc));
    g.zc = (int)(zc > 0 ? zc : 1);
  }
  g.rz = s.nz > 1; g.ry = s.ny > 1; g.rx = s.nx > 1;
  // persistent in-plane grid: the resident block count (3 per SM for TM <= 10, else 2)
  // (tile height and blocks per SM as pl_ty / pl_bps of the lag template chosen for T)
  const int ty = (sizeof(E) == 4 && T <= 10) ? 64 : 32;
  const int64_t W = cdiv(s.nx, kPlTX) * cdiv(s.ny, ty) * nzo;
  const int64_t G = (int64_t)sm_count() * (ty == 64 ? 2 : (T <= 10 ? 3 : 2));
  g.pzc = 0;
  g.z = dim3((unsigned)cdiv(s.nx, kTX), (unsigned)cdiv(s.ny, kTY), (unsigned)cdiv(nzo, g.zc));
  {  // persistent TMA z-walk: the resident block count (register bound 3 / 2 per SM, shared-memory bound)
    const int tm = T <= 10 ? (T + 1) / 2 * 2 : (T <= 12 ? 12 : 16), cpt = kWalkCPT<E>;
    const int64_t smem = (int64_t)2 * tm * cpt * kWalkThreads * 2 * (int64_t)sizeof(E) + 2 * tm * 8 + 16 +
                         (int64_t)tm * kWalkThreads * 8 + 1024;
    int64_t bps = (227 * 1024 + 1024) / smem;
    const int64_t rb = cpt == 1 ? 3 : 2;
    if (bps > rb) bps = rb;
    if (bps < 1) bps = 1;
    const int64_t Wz = cdiv(s.nx, kWalkCPT<E> * kWalkThreads) * s.ny * nzo, Gz = (int64_t)sm_count() * bps;
    g.zt = dim3((unsigned)(Wz < Gz ? Wz : Gz), 1, 1);
  }
  g.pl = dim3((unsigned)(W < G ? W : G), 1, 1);
  g.x = dim3((unsigned)cdiv(nzo * s.ny, kXWarps * 32), (unsigned)cdiv(s.nx, g.xc), 1);
  g.xvec = dim3((unsigned)cdiv(nzo * s.ny, 256), (unsigned)cdiv(s.nx, g.xc), 1);
  return g;
}
template <typename E>
int64_t ac_blocks(const Field3<E>& s, int T) {
  const AcGrids g = ac_grids(s, T);
  auto n = [](dim3 d) { return (int64_t)d.x * d.y * d.z; };
  auto mx = [](int64_t a, int64_t b) { return a > b ? a : b; };
  return mx(n(g.z), n(g.zt)) + n(g.pl) + mx(n(g.x), n(g.xvec));
}

template <typename E, int TM>
static cudaError_t launch_ac_t(const Field3<E>& s, int T, double* parts, DevResults* res,
                               unsigned int* tickets, cudaStream_t st) {
  const AcGrids g = ac_grids(s, T);
  auto n = [](dim3 d) { return (size_t)d.x * d.y * d.z; };
  // rows 16-byte aligned (nx * sizeof(E) % 16 == 0, aligned segments): TMA bulk-copy z-walk and
  // 16-byte plane staging; the vector x-walk (1-D fields) is float32 only
  bool vec = (s.nx * (int64_t)sizeof(E)) % 16 == 0;
  for (int k = 0; k < s.nseg; k++)
    vec = vec && (reinterpret_cast<uintptr_t>(s.xs[k]) % 16) == 0 && (reinterpret_cast<uintptr_t>(s.ys[k]) % 16) == 0;
  double* pz = parts;
  double* pp = pz + (vec ? n(g.zt) : n(g.z)) * kAcSlots;
  double* px = pp + n(g.pl) * kAcSlots;
  cudaError_t e = cudaMemsetAsync(res->rec.ac, 0, sizeof(res->rec.ac), st);
  if (e != cudaSuccess) return e;
  if (g.rz && vec) {
    constexpr int C = kWalkCPT<E>;
    constexpr int wsm = zwalk_smem<E, TM, C>();
    if ((e = set_smem_once<ac_zwalk_tma<E, TM, C>>(wsm)) != cudaSuccess) return e;
    ac_zwalk_tma<E, TM, C><<<g.zt, kWalkThreads, wsm, st>>>(s, T, g.zc, pz, res, tickets + 0);
  } else if (g.rz) {
    ac_zwalk<E, TM><<<g.z, dim3(kTX, kTY), 0, st>>>(s, T, g.zc, pz, res, tickets + 0);
  }
  if (g.ry) {
    constexpr int psm = (int)sizeof(PlaneTile<E, TM>);
    // 16-byte staging needs aligned rows; tile-relative offsets are 32-bit
    const bool pvec = vec && (int64_t)(pl_ty<E, TM>() + TM) * s.nx < ((int64_t)1 << 31);
    static const CUtensorMap no_map{};
    bool done = false;
#if CZC_AC_TMA
    if constexpr (sizeof(E) == 4) {
      // the windows arrive by tensor copies; the owned planes lie in one segment (the whole field,
      // or the local slab in slab mode, whose halo planes the in-plane lags never read): map it
      int seg = -1;
      for (int k = 0; k < s.nseg; k++)
        if (s.zs[k] <= s.zown0 && s.zown1 <= s.zs[k + 1]) seg = k;
      if (pvec && seg >= 0) {
        using PT = PlaneTile<E, TM>;
        CUtensorMap mx, my;
        const int64_t nzs = s.zs[seg + 1] - s.zs[seg];
        if (encode_plane_map(&mx, s.xs[seg], s.nx, s.ny, nzs, PT::PF, PT::HY) &&
            encode_plane_map(&my, s.ys[seg], s.nx, s.ny, nzs, PT::PF, PT::HY)) {
          if ((e = set_smem_once<ac_plane<E, TM, true, true>>(psm)) != cudaSuccess) return e;
          ac_plane<E, TM, true, true><<<g.pl, kPlThreads, psm, st>>>(s, pp, res, tickets + 1, mx, my, s.zs[seg]);
          done = true;
        }
      }
    }
#endif
    if (!done) {
      auto kern = pvec ? ac_plane<E, TM, true, false> : ac_plane<E, TM, false, false>;
      if ((e = pvec ? set_smem_once<ac_plane<E, TM, true, false>>(psm) : set_smem_once<ac_plane<E, TM, false, false>>(psm)) !=
          cudaSuccess)
        return e;
      kern<<<g.pl, kPlThreads, psm, st>>>(s, pp, res, tickets + 1, no_map, no_map, 0);
    }
  } else if (g.rx) {
    bool done = false;
    if constexpr (sizeof(E) == 4) {
      if (vec) {
        ac_xwalk_vec<TM><<<g.xvec, 256, 0, st>>>(s, T, g.xc, px, res, tickets + 2);
        done = true;
      }
    }
    if (!done) ac_xwalk_smem<E, TM><<<g.x, kXWarps * 32, 0, st>>>(s, T, g.xc, px, res, tickets + 2);
  }
  return cudaGetLastError();
}

// tickets: three consecutive counters (z, y, x walks)
template <typename E>
cudaError_t launch_ac(const Field3<E>& s, int T, int, double* parts, DevResults* res,
                      unsigned int* tickets, cudaStream_t st) {
  if (T <= 2) return launch_ac_t<E, 2>(s, T, parts, res, tickets, st);
  if (T <= 4) return launch_ac_t<E, 4>(s, T, parts, res, tickets, st);
  if (T <= 6) return launch_ac_t<E, 6>(s, T, parts, res, tickets, st);
  if (T <= 8) return launch_ac_t<E, 8>(s, T, parts, res, tickets, st);
  if (T <= 10) return launch_ac_t<E, 10>(s, T, parts, res, tickets, st);
  if (T <= 12) return launch_ac_t<E, 12>(s, T, parts, res, tickets, st);
  return launch_ac_t<E, 16>(s, T, parts, res, tickets, st);
}

#define CZC_P2_INST(E)                                                                              \
  template int64_t deriv_blocks<E>(const Field3<E>&, int);                                          \
  template int64_t ac_blocks<E>(const Field3<E>&, int);                                             \
  template cudaError_t launch_deriv<E>(const Field3<E>&, int, double*, DevResults*, unsigned int*,  \
                                       double*, cudaStream_t);                                      \
  template cudaError_t launch_ac<E>(const Field3<E>&, int, int, double*, DevResults*, unsigned int*, \
                                    cudaStream_t);
CZC_P2_INST(float)
CZC_P2_INST(double)
#undef CZC_P2_INST

}  // namespace czc

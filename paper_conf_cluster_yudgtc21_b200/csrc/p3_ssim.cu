// p3_ssim.cu — Pattern 3: sliding-window SSIM.
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
//   (a) z-walk — keeps FP64 running sums over the last WZ planes of four anchored moments
//         a = x - K,  e = y - x,  a*b (b = y - K),  e*e
//       in registers; the leaving plane's x sits in a per-thread register ring (the paper's
//       FIFO, moved from window partials to raw samples; a shifting ring, so the plane loop
//       needs no unrolling), which also gives the z-window min/max of x, and its
//       y is re-read from L2; the next plane is prefetched into registers one plane ahead;
//   (b) y-pass — after ONE __syncthreads on a double-buffered shared-memory exchange of the
//       z-sums, each warp forms running sums over WY rows for its G origin rows;
//   (c) x-pass — power-of-two doubling with warp shuffles across the 32 lanes (the paper's
//       shfl_down x-reduction, L270), then the per-window mix in the cancellation-free form
//         ssim = A/(A + mu_e^2) * B/(B + s_e^2),  A = 2 mu_x mu_y + C1,  B = 2 s_xy + C2
//       (identical to Wang et al.'s formula with C3 = C2/2, reading R14), with L = max - min of
//       the original window (reading R15) or the global range.
// K is one anchor per block (the tile-centre sample of its first plane) so the moment sums stay
// small; every sum is FP64.  Window extents are compile-time (cubic 3-D, square 2-D, 1-D).
#include "czc_internal.cuh"

namespace czc {

constexpr int kP3Warps = 8;
constexpr int kP3Threads = 32 * kP3Warps;

template <typename T, int WX, int WY, int WZ, int G>
struct SsimGeom {
  static constexpr int TX = 32 - WX + 1;                 // origins per tile along x
  static constexpr int TY = kP3Warps * G;                // origins per tile along y
  static constexpr int FY = TY + WY - 1;                 // footprint rows
  static constexpr int KC = (FY + kP3Warps - 1) / kP3Warps;   // z-walk rows per thread
  static constexpr int ZSTRIDE = FY * 32;                // one component plane of the exchange
  // exchange buffer: { 4 double comps, 2 min/max comps of the input type } x FY x 32, double-buffered
  static constexpr size_t buf_bytes = (size_t)ZSTRIDE * (4 * sizeof(double) + 2 * sizeof(T));
  static constexpr size_t smem = 2 * buf_bytes;
};

__device__ __forceinline__ double shd(double v, int d) { return __shfl_down_sync(0xffffffffu, v, d); }
__device__ __forceinline__ float shf(float v, int d) { return __shfl_down_sync(0xffffffffu, v, d); }

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

// T = float: the x ring and the exchanged extrema are floats (exact); T = double: doubles, one
// block per SM for the larger register ring.
template <typename T, int WX, int WY, int WZ, int G>
__global__ void __launch_bounds__(kP3Threads, (kP3Warps <= 8 && SsimGeom<T, WX, WY, WZ, G>::KC * WZ * sizeof(T) <= 128) ? 2 : 1)
p3_kernel(Field3<T> f, SsimParams p, double* __restrict__ parts, DevResults* __restrict__ res,
          unsigned int* __restrict__ ticket, double* __restrict__ dbg) {
  using Gm = SsimGeom<T, WX, WY, WZ, G>;
  constexpr int TX = Gm::TX, FY = Gm::FY, KC = Gm::KC, ZS = Gm::ZSTRIDE;
  constexpr double invM = 1.0 / (double)(WX * WY * WZ);
  extern __shared__ __align__(16) unsigned char smem_raw[];

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
  const double K = (zb < zend) ? (double)f.xp(zb)[ky * f.nx + kx] : 0.0;
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
  auto load = [&](int n, bool has_old) {                 // has_old: n >= WZ (constant per call site)
    if (n < nsteps) {                                    // block-uniform
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
  };

  double sm[KC][4];
  T ring[KC][WZ];                                        // x of the last WZ planes
#pragma unroll
  for (int k = 0; k < KC; k++) {
#pragma unroll
    for (int m = 0; m < 4; m++) sm[k][m] = 0;
#pragma unroll
    for (int s = 0; s < WZ; s++) ring[k][s] = 0;
  }
  load(0, false);

  double ssum = 0;
  unsigned scnt = 0;
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

  // One plane step; warm = (step >= WZ: a plane leaves the z-window) and, in the warm-up, s =
  // step are compile-time constants at every call site, so the warm-up planes carry no per-step
  // tests.
  auto step_body = [&](const int step, const int s, const bool warm) {
    // the prefetched plane is consumed by the z-walk below, then the next one is requested
    // into the same registers (no copies; its latency hides behind the y / x passes)
    const int buf = step & 1;
    double* Zd = reinterpret_cast<double*>(smem_raw + buf * Gm::buf_bytes);
    T* Zm = reinterpret_cast<T*>(Zd + 4 * ZS);
    const bool full = warm || s == WZ - 1;               // a complete z-window ends here
    // ---- (a) z-walk --------------------------------------------------------------------
#pragma unroll
    for (int k = 0; k < KC; k++) {
      if (!row_live(k)) continue;
      {
        const double xd = nxt[k].x, yd = nxt[k].y;
        const double a = xd - K, b = yd - K, e = yd - xd;
        sm[k][0] += a; sm[k][1] += e; sm[k][2] = fma(a, b, sm[k][2]); sm[k][3] = fma(e, e, sm[k][3]);
      }
      if (warm) {
        const double xd = ring[k][0], yd = nyo[k];
        const double a = xd - K, b = yd - K, e = yd - xd;
        sm[k][0] -= a; sm[k][1] -= e; sm[k][2] = fma(-a, b, sm[k][2]); sm[k][3] = fma(-e, e, sm[k][3]);
      }
      // shifting ring (oldest plane first; WZ - 1 register moves per row): the main loop is not
      // unrolled, so one copy of the step (~4.4 K instructions for the kernel instead of 10.3 K
      // with a static-slot ring unrolled by WZ) stays in the instruction cache — the
      // `no_instruction` stalls of the unrolled version cost more than the moves (0.475 -> 0.445 ms)
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
      }
    }
    load(step + 1, warm || s == WZ - 1);
    if (!full) return;                                   // no complete z-window yet
    __syncthreads();
    const bool zok = zph == 0;                           // origin plane zb + step - WZ + 1
    zph = zph + 1 == p.sz ? 0 : zph + 1;
    // ---- (b) y-pass: the G origin rows of this warp (running sums over WY rows) ------------
    double h[G][4];
    T hmn[G], hmx[G];
    {
      // y-window min/max: the WY - G + 1 rows shared by all G windows are reduced once
      T cmn = Zm[(warp * G + G - 1) * 32 + lane], cmx = Zm[ZS + (warp * G + G - 1) * 32 + lane];
#pragma unroll
      for (int i = G; i < WY; i++) {
        cmn = tmin(cmn, Zm[(warp * G + i) * 32 + lane]);
        cmx = tmax(cmx, Zm[ZS + (warp * G + i) * 32 + lane]);
      }
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
      // A, B, A + mu_e^2, B + s_e^2 > 0 (C1, C2 > 0); |rel err of the reciprocal| <= 2u
      const double ssim = (A * B) * fast_rcp((A + mue * mue) * (B + see));
      ssum += ok ? ssim : 0.0;
      scnt += ok ? 1u : 0u;
      if (dbg && ok) {
        const int64_t oz = zb + step - WZ + 1, gy = y0 + warp * G + g;
        dbg[((oz / p.sz) * p.nwy + gy / p.sy) * p.nwx + (x0 + lane) / p.sx] = ssim;
      }
    }
  };

  // warm-up: planes 0 .. WZ-1 (the last one completes the first z-window)
#pragma unroll
  for (int s = 0; s < WZ; s++) {
    if (s >= nsteps) break;                              // block-uniform
    step_body(s, s, false);
  }
#pragma unroll 1
  for (int step = WZ; step < nsteps; step++) step_body(step, 0, true);

  double rec[kSsimSlots] = {ssum, (double)scnt, 0.0};
  const unsigned bid = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
  struct Sum { __device__ int operator()(int) const { return OP_SUM; } };
  __syncthreads();
  block_reduce_slots<kSsimSlots>(rec, Sum{}, parts + (size_t)bid * kSsimSlots);
  if (!last_block_arrive(ticket)) return;
  finish_slots<kSsimSlots>(parts, gridDim.x * gridDim.y * gridDim.z, Sum{}, res->rec.ssim);
  if (tid == 0) *ticket = 0;
}

static inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

template <typename T, int WX, int WY, int WZ, int G>
static cudaError_t launch_t(const Field3<T>& f, const SsimParams& p, double* parts,
                            DevResults* res, unsigned int* ticket, double* dbg, cudaStream_t st,
                            int64_t* nblocks_out) {
  using Gm = SsimGeom<T, WX, WY, WZ, G>;
  auto kern = p3_kernel<T, WX, WY, WZ, G>;
  cudaError_t e = set_smem_once<p3_kernel<T, WX, WY, WZ, G>>((int)Gm::smem);
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
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kP3Threads, Gm::smem) != cudaSuccess || occ < 1) occ = 1;
  }
  const int64_t slots = (int64_t)(sms > 0 ? sms : 148) * occ;
  const int64_t n0 = cdiv(noz, p.zchunk);
  int64_t best_n = n0, best_cost = INT64_MAX;
  for (int64_t nch = n0 > 2 ? n0 - 2 : 1; nch <= n0 + 2 && nch <= noz; nch++) {
    const int64_t zc = cdiv(noz, nch);
    if (cdiv(noz, zc) != nch) continue;               // the same chunking as a smaller count
    const int64_t cost = cdiv(tiles * nch, slots) * (zc + WZ - 1);
    if (cost < best_cost) { best_cost = cost; best_n = nch; }
  }
  SsimParams q = p;
  q.zchunk = (int)cdiv(noz, best_n);
  dim3 grid((unsigned)cdiv(f.nx - WX + 1, Gm::TX), (unsigned)cdiv(f.ny - WY + 1, Gm::TY),
            (unsigned)cdiv(noz, q.zchunk));
  if (nblocks_out) { *nblocks_out = (int64_t)grid.x * grid.y * grid.z; return cudaSuccess; }
  if (f.ny * f.nx >= (int64_t)1 << 31) return cudaErrorInvalidValue;   // 32-bit in-plane offsets
  kern<<<grid, kP3Threads, Gm::smem, st>>>(f, q, parts, res, ticket, dbg);
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// 2-D fields (square W x W windows): the rows stream like the planes of the 3-D kernel, and the
// y-window is the running sum of that stream, so no shared-memory exchange and no barrier are
// needed: warp w of a block owns its own tile of 32 - W + 1 x-origins (lane = footprint column),
// keeps FP64 running sums of the four anchored moments over the last W rows plus the rows' x in
// a shifting register ring (warm-up peeled), re-reads the leaving row's y from L2, and
// per row does the x-pass by shuffles and the mix.  (The 3-D kernel on a one-plane field ran one
// plane per block: 0.29 ms for the 1800 x 3600 CESM-shaped pair.)
constexpr int kRowWarps = 8;
template <typename T, int W>
__global__ void __launch_bounds__(kRowWarps * 32)
p3_rows_kernel(Field3<T> f, SsimParams p, int rchunk, double* __restrict__ parts, DevResults* __restrict__ res,
               unsigned int* __restrict__ ticket, double* __restrict__ dbg) {
  constexpr int TX = 32 - W + 1;
  constexpr double invM = 1.0 / (double)(W * W);
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
  const double K = (double)X[ky * nx + kx];                     // anchor of this warp's tile
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
  double sm0 = 0, sm1 = 0, sm2 = 0, sm3 = 0;
  T ring[W];
#pragma unroll
  for (int t = 0; t < W; t++) ring[t] = 0;
  double ssum = 0;
  unsigned scnt = 0;
  int rph = (int)(rb % p.sy);
  load(0, false);
  auto step_body = [&](const int step, const int s, const bool warm) {
    const bool full = warm || s == W - 1;
    {
      const double xd = nx_, yd = ny_;
      const double a = xd - K, b = yd - K, e = yd - xd;
      sm0 += a; sm1 += e; sm2 = fma(a, b, sm2); sm3 = fma(e, e, sm3);
    }
    if (warm) {
      const double xd = ring[0], yd = nyo;
      const double a = xd - K, b = yd - K, e = yd - xd;
      sm0 -= a; sm1 -= e; sm2 = fma(-a, b, sm2); sm3 = fma(-e, e, sm3);
    }
#pragma unroll
    for (int t = 0; t + 1 < W; t++) ring[t] = ring[t + 1];     // shifting ring, oldest first
    ring[W - 1] = nx_;
    load(step + 1, warm || s == W - 1);
    if (!full) return;
    T mn = ring[0], mx = ring[0];
#pragma unroll
    for (int t = 1; t < W; t++) { mn = tmin(mn, ring[t]); mx = tmax(mx, ring[t]); }
    const double S0 = lane_window_sum<W>(sm0), S1 = lane_window_sum<W>(sm1);
    const double S2 = lane_window_sum<W>(sm2), S3 = lane_window_sum<W>(sm3);
    const T wmn = lane_window_ext<W, false>(mn), wmx = lane_window_ext<W, true>(mx);
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
    const double ssim = (A * B) * fast_rcp((A + mue * mue) * (B + see));
    ssum += ok ? ssim : 0.0;
    scnt += ok ? 1u : 0u;
    if (dbg && ok) dbg[((rb + step - W + 1) / p.sy) * p.nwx + gx / p.sx] = ssim;
  };
#pragma unroll
  for (int s = 0; s < W; s++) {
    if (s >= nsteps) break;                                     // block-uniform
    step_body(s, s, false);
  }
#pragma unroll 1
  for (int step = W; step < nsteps; step++) step_body(step, 0, true);
  double rec[kSsimSlots] = {ssum, (double)scnt, 0.0};
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

// p3_ssim.cu — Pattern 3: sliding-window SSIM.
//
// Paper (L139-L146, Fig. 5, Alg. 3): a w^3 window slides with a fixed step over both
// fields; at each position the window's min, max, sum and power sums are reduced, "mixed (by some
// simple sums and multiplications) to generate the local SSIM", and a global reduction averages
// the local SSIMs.  The paper's kernel keeps per-slice window partials in a shared-memory FIFO of
// depth w along z so each slice is "read and processed only once" (L270, L318).
//
// B200 design.  A block owns a tile of 32 (x) x 8 (y) window origins and a chunk
// of origin planes, and streams z:
//   (a) z-walk: every thread owns footprint columns (y, x) of the tile + halo and keeps FP64
//       running sums over the last WZ planes of the four anchored moments
//         a = x - K,  e = y - x,  a*b (b = y - K),  e*e
//       (the leaving plane comes from a shared-memory ring of raw (x, y) — the paper's FIFO moved
//       from window partials to raw samples), plus the z-window min / max of x from the ring;
//   (b) y-pass: running sums over WY rows, segments of 4 origins per thread;
//   (c) x-pass: running sums over WX columns, then the per-window mix in the cancellation-free
//       two-factor form  ssim = A/(A + mu_e^2) * B/(B + s_e^2),  A = 2 mu_x mu_y + C1,
//       B = 2 s_xy + C2  (identical to Wang et al.'s formula with C3 = C2/2, reading R14), with
//       L = max - min of the original window (reading R15) or the global range.
// K is one anchor per block (the tile-centre sample of its first plane) so the moment sums stay
// small; all sums are FP64.  Window extents are compile-time (cubic 3-D, square 2-D, or 1-D).
#include "czc_internal.cuh"

namespace czc {

constexpr int kOX = 32;     // origins per tile along x
constexpr int kOY = 8;      // origins per tile along y
constexpr int kSeg = 4;     // origins per thread in the running-sum passes
constexpr int kP3Threads = 256;

template <int WY, int WX, int WZ>
struct SsimGeom {
  static constexpr int FX = kOX + WX - 1;
  static constexpr int FY = kOY + WY - 1;
  static constexpr int NCOL = FX * FY;
  static constexpr int KC = (NCOL + kP3Threads - 1) / kP3Threads;
  static constexpr size_t ring_bytes = (size_t)WZ * NCOL * sizeof(float2);
  static constexpr size_t z_bytes = (size_t)NCOL * (4 * sizeof(double) + 2 * sizeof(float));
  static constexpr size_t h_bytes = (size_t)kOY * FX * (4 * sizeof(double) + 2 * sizeof(float));
  static constexpr size_t smem = ring_bytes + z_bytes + h_bytes;
};

template <int WY, int WX, int WZ>
__global__ void __launch_bounds__(kP3Threads)
p3_kernel(Field3 f, SsimParams p,
          double* __restrict__ parts, DevResults* __restrict__ res, unsigned int* __restrict__ ticket,
          double* __restrict__ dbg) {
  using G = SsimGeom<WY, WX, WZ>;
  constexpr int FX = G::FX, FY = G::FY, NCOL = G::NCOL, KC = G::KC;
  constexpr double invM = 1.0 / (double)(WX * WY * WZ);
  extern __shared__ __align__(16) unsigned char smem_raw[];
  float2* ring = reinterpret_cast<float2*>(smem_raw);                       // [WZ][NCOL]
  double* Zd = reinterpret_cast<double*>(smem_raw + G::ring_bytes);         // [4][NCOL]
  float* Zm = reinterpret_cast<float*>(Zd + 4 * NCOL);                      // [2][NCOL]
  double* Hd = reinterpret_cast<double*>(smem_raw + G::ring_bytes + G::z_bytes);  // [4][kOY][FX]
  float* Hm = reinterpret_cast<float*>(Hd + 4 * kOY * FX);                  // [2][kOY][FX]

  const int tid = threadIdx.x;
  const int64_t x0 = (int64_t)blockIdx.x * kOX, y0 = (int64_t)blockIdx.y * kOY;
  const int64_t zb = f.zown0 + (int64_t)blockIdx.z * p.zchunk;
  int64_t zo_end = zb + p.zchunk;                        // origin planes [zb, zo_end)
  if (zo_end > f.zown1) zo_end = f.zown1;
  if (zo_end > f.nz - WZ + 1) zo_end = f.nz - WZ + 1;

  // anchor: tile-centre sample of the first plane (clamped into the field)
  int64_t ky = y0 + FY / 2, kx = x0 + FX / 2;
  if (ky > f.ny - 1) ky = f.ny - 1;
  if (kx > f.nx - 1) kx = f.nx - 1;
  const double K = (zb < zo_end) ? (double)f.xp(zb)[ky * f.nx + kx] : 0.0;
  const double Lglob = (double)res->p1.xmax - (double)res->p1.xmin;

  // per-thread footprint columns and their running z-sums
  double rs[KC][4];
  int64_t cofs[KC];
  bool cin[KC];
#pragma unroll
  for (int k = 0; k < KC; k++) {
    const int c = tid + k * kP3Threads;
    const int r = c / FX, cc = c % FX;
    const int64_t gy = y0 + r, gx = x0 + cc;
    cin[k] = c < NCOL && gy < f.ny && gx < f.nx;
    cofs[k] = cin[k] ? gy * f.nx + gx : 0;
#pragma unroll
    for (int m = 0; m < 4; m++) rs[k][m] = 0;
  }

  double ssum = 0, scnt = 0;
  const int64_t zplanes_end = (zo_end > zb) ? zo_end + WZ - 1 : zb;
  for (int64_t zi = zb; zi < zplanes_end; zi++) {
    const int step = (int)(zi - zb);
    const int slot = step % WZ;
    const float* Xz = f.xp(zi);
    const float* Yz = f.yp(zi);
    // ---- (a) z-walk ------------------------------------------------------------------------
#pragma unroll
    for (int k = 0; k < KC; k++) {
      const int c = tid + k * kP3Threads;
      if (c < NCOL) {
        float xv = 0.f, yv = 0.f;
        if (cin[k]) { xv = Xz[cofs[k]]; yv = Yz[cofs[k]]; }
        float2* rp = ring + (size_t)slot * NCOL + c;
        {
          const double xd = xv, yd = yv;
          const double a = xd - K, b = yd - K, e = yd - xd;
          rs[k][0] += a; rs[k][1] += e; rs[k][2] = fma(a, b, rs[k][2]); rs[k][3] = fma(e, e, rs[k][3]);
        }
        if (step >= WZ) {
          const float2 o = *rp;
          const double xd = o.x, yd = o.y;
          const double a = xd - K, b = yd - K, e = yd - xd;
          rs[k][0] -= a; rs[k][1] -= e; rs[k][2] = fma(-a, b, rs[k][2]); rs[k][3] = fma(-e, e, rs[k][3]);
        }
        *rp = make_float2(xv, yv);
        if (step >= WZ - 1) {
          float mn = xv, mx = xv;
#pragma unroll
          for (int s = 0; s < WZ; s++) {
            const float v = ring[(size_t)s * NCOL + c].x;
            mn = fminf(mn, v);
            mx = fmaxf(mx, v);
          }
#pragma unroll
          for (int m = 0; m < 4; m++) Zd[m * NCOL + c] = rs[k][m];
          Zm[c] = mn;
          Zm[NCOL + c] = mx;
        }
      }
    }
    if (step < WZ - 1) continue;           // no complete z-window yet (block-uniform)
    const int64_t oz = zi - WZ + 1;        // origin plane of the windows completed now
    __syncthreads();
    // ---- (b) y-pass: columns of Z, running sums over WY rows --------------------------------
    for (int item = tid; item < FX * (kOY / kSeg); item += kP3Threads) {
      const int cx = item % FX, oy0 = (item / FX) * kSeg;
#pragma unroll
      for (int m = 0; m < 4; m++) {
        double v[kSeg + WY - 1];
#pragma unroll
        for (int i = 0; i < kSeg + WY - 1; i++) v[i] = Zd[m * NCOL + (oy0 + i) * FX + cx];
        double s = 0;
#pragma unroll
        for (int i = 0; i < WY; i++) s += v[i];
        Hd[(m * kOY + oy0) * FX + cx] = s;
#pragma unroll
        for (int j = 1; j < kSeg; j++) {
          s += v[j + WY - 1] - v[j - 1];
          Hd[(m * kOY + oy0 + j) * FX + cx] = s;
        }
      }
      float vn[kSeg + WY - 1], vx[kSeg + WY - 1];
#pragma unroll
      for (int i = 0; i < kSeg + WY - 1; i++) {
        vn[i] = Zm[(oy0 + i) * FX + cx];
        vx[i] = Zm[NCOL + (oy0 + i) * FX + cx];
      }
#pragma unroll
      for (int j = 0; j < kSeg; j++) {
        float mn = vn[j], mx = vx[j];
#pragma unroll
        for (int i = 1; i < WY; i++) { mn = fminf(mn, vn[j + i]); mx = fmaxf(mx, vx[j + i]); }
        Hm[(oy0 + j) * FX + cx] = mn;
        Hm[(kOY + oy0 + j) * FX + cx] = mx;
      }
    }
    __syncthreads();
    // ---- (c) x-pass + mix -------------------------------------------------------------------
    const bool zok = (oz % p.sz) == 0;
    for (int item = tid; item < kOY * (kOX / kSeg); item += kP3Threads) {
      const int oy = item / (kOX / kSeg), ox0 = (item % (kOX / kSeg)) * kSeg;
      double S[4][kSeg];
#pragma unroll
      for (int m = 0; m < 4; m++) {
        double v[kSeg + WX - 1];
#pragma unroll
        for (int i = 0; i < kSeg + WX - 1; i++) v[i] = Hd[(m * kOY + oy) * FX + ox0 + i];
        double s = 0;
#pragma unroll
        for (int i = 0; i < WX; i++) s += v[i];
        S[m][0] = s;
#pragma unroll
        for (int j = 1; j < kSeg; j++) { s += v[j + WX - 1] - v[j - 1]; S[m][j] = s; }
      }
      float vn[kSeg + WX - 1], vx[kSeg + WX - 1];
#pragma unroll
      for (int i = 0; i < kSeg + WX - 1; i++) {
        vn[i] = Hm[oy * FX + ox0 + i];
        vx[i] = Hm[(kOY + oy) * FX + ox0 + i];
      }
      const int64_t gy = y0 + oy;
      const bool yok = gy <= f.ny - WY && (gy % p.sy) == 0;
#pragma unroll
      for (int j = 0; j < kSeg; j++) {
        const int64_t gx = x0 + ox0 + j;
        if (!(zok && yok && gx <= f.nx - WX && (gx % p.sx) == 0)) continue;
        float mn = vn[j], mx = vx[j];
#pragma unroll
        for (int i = 1; i < WX; i++) { mn = fminf(mn, vn[j + i]); mx = fmaxf(mx, vx[j + i]); }
        const double mua = S[0][j] * invM, mue = S[1][j] * invM;
        const double mux = K + mua, muy = mux + mue;
        const double sxy = S[2][j] * invM - mua * (mua + mue);
        const double see = S[3][j] * invM - mue * mue;
        double L = p.range_mode ? Lglob : (double)mx - (double)mn;
        if (L == 0) L = 1.0;
        const double C1 = (0.01 * L) * (0.01 * L), C2 = (0.03 * L) * (0.03 * L);
        const double A = 2.0 * mux * muy + C1, B = 2.0 * sxy + C2;
        const double ssim = (A * B) / ((A + mue * mue) * (B + see));
        ssum += ssim;
        scnt += 1.0;
        if (dbg) dbg[((oz / p.sz) * p.nwy + gy / p.sy) * p.nwx + gx / p.sx] = ssim;
      }
    }
    // the next (a) only writes the ring / Z, which (c) does not read; (b) of the next plane is
    // behind the __syncthreads after that (a), so H is not overwritten while (c) reads it.
  }

  double rec[kSsimSlots] = {ssum, scnt, 0.0};
  const unsigned bid = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
  struct Sum { __device__ int operator()(int) const { return OP_SUM; } };
  block_reduce_slots<kSsimSlots>(rec, Sum{}, parts + (size_t)bid * kSsimSlots);
  if (!last_block_arrive(ticket)) return;
  finish_slots<kSsimSlots>(parts, gridDim.x * gridDim.y * gridDim.z, Sum{}, res->ssim);
  if (tid == 0) *ticket = 0;
}

static inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

template <int WY, int WX, int WZ>
static cudaError_t launch_t(const Field3& f, const SsimParams& p, double* parts,
                            DevResults* res, unsigned int* ticket, double* dbg, cudaStream_t st,
                            int64_t* nblocks_out) {
  using G = SsimGeom<WY, WX, WZ>;
  int64_t zhi = f.zown1 < f.nz - WZ + 1 ? f.zown1 : f.nz - WZ + 1;
  const int64_t noz = zhi > f.zown0 ? zhi - f.zown0 : 1;
  dim3 grid((unsigned)cdiv(f.nx - WX + 1, kOX), (unsigned)cdiv(f.ny - WY + 1, kOY), (unsigned)cdiv(noz, p.zchunk));
  if (nblocks_out) { *nblocks_out = (int64_t)grid.x * grid.y * grid.z; return cudaSuccess; }
  cudaError_t e = cudaFuncSetAttribute(p3_kernel<WY, WX, WZ>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)G::smem);
  if (e != cudaSuccess) return e;
  p3_kernel<WY, WX, WZ><<<grid, kP3Threads, G::smem, st>>>(f, p, parts, res, ticket, dbg);
  return cudaGetLastError();
}

// Dispatch on the (compile-time) window: cubic (3-D), square (2-D, WZ = 1) or 1-D (WY = WZ = 1).
template <int W>
static cudaError_t dispatch_w(int kind, const Field3& f, const SsimParams& p, double* parts,
                              DevResults* res, unsigned int* ticket, double* dbg, cudaStream_t st, int64_t* nb) {
  if (kind == 3) return launch_t<W, W, W>(f, p, parts, res, ticket, dbg, st, nb);
  if (kind == 2) return launch_t<W, W, 1>(f, p, parts, res, ticket, dbg, st, nb);
  return launch_t<1, W, 1>(f, p, parts, res, ticket, dbg, st, nb);
}

// kind: 3 = (W,W,W) cubic window, 2 = (W,W) with z inactive, 1 = x only.  Returns
// cudaErrorInvalidValue for unsupported W.  If nblocks_out != NULL only the grid size is returned.
cudaError_t launch_ssim(int kind, int W, const Field3& f, const SsimParams& p,
                        double* parts, DevResults* res, unsigned int* ticket, double* dbg,
                        cudaStream_t st, int64_t* nblocks_out) {
  switch (W) {
#define CZC_W(w) case w: return dispatch_w<w>(kind, f, p, parts, res, ticket, dbg, st, nblocks_out);
    CZC_W(2) CZC_W(3) CZC_W(4) CZC_W(5) CZC_W(6) CZC_W(7) CZC_W(8) CZC_W(9) CZC_W(10)
    CZC_W(11) CZC_W(12) CZC_W(13) CZC_W(14) CZC_W(15) CZC_W(16)
#undef CZC_W
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace czc

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
// B200 design: blocks own a 32 x 8 (x, y) column tile and stream along z; the
// z-neighbours live in registers, the in-plane neighbours in a shared-memory plane with halo;
// per-thread FP64 accumulators; block partials combined by the last block in index order.
#include "czc_internal.cuh"

namespace czc {

constexpr int kTX = 32, kTY = 8;

__device__ __forceinline__ void deriv_fields(const double c, const double zp, const double zm,
                                             const double yp, const double ym, const double xp,
                                             const double xm, bool az, bool ay, bool ax,
                                             double F[CZC_NDERIV]) {
  double der1 = 0, der2 = 0, g2 = 0, div = 0, lap = 0;
  // axis order z, y, x (slowest first) — same as the oracle
#define CZC_AXIS(ACT, P, M)                     \
  if (ACT) {                                    \
    const double delta = (P) - (M);             \
    const double D = delta / 2.0;               \
    const double l = (P) - 2.0 * c + (M);       \
    der1 += fabs(delta);                        \
    der2 += fabs(l);                            \
    g2 += D * D;                                \
    div += D;                                   \
    lap += l;                                   \
  }
  CZC_AXIS(az, zp, zm)
  CZC_AXIS(ay, yp, ym)
  CZC_AXIS(ax, xp, xm)
#undef CZC_AXIS
  F[CZC_DER1] = der1;
  F[CZC_DER2] = der2;
  F[CZC_GRAD] = sqrt(g2);
  F[CZC_DIV] = div;
  F[CZC_LAP] = lap;
}

struct DerivOp {
  __device__ int operator()(int k) const { return deriv_op(k); }
};
struct SumOp {
  __device__ int operator()(int) const { return OP_SUM; }
};

// grid: (ceil(nx/32), ceil(ny/8), nzchunks); block (32, 8)
__global__ void __launch_bounds__(kTX * kTY)
deriv_kernel(Field3 s, int zchunk,
             double* __restrict__ parts, DevResults* __restrict__ res, unsigned int* __restrict__ ticket) {
  __shared__ double sx[kTY + 2][kTX + 2];
  __shared__ double sy[kTY + 2][kTX + 2];
  const int tx = threadIdx.x, ty = threadIdx.y, tid = ty * kTX + tx;
  const int64_t gx = (int64_t)blockIdx.x * kTX + tx, gy = (int64_t)blockIdx.y * kTY + ty;
  const bool az = s.nz > 1, ay = s.ny > 1, ax = s.nx > 1;
  const int64_t plane = s.ny * s.nx;
  // interior ranges (reading R11)
  int64_t zlo = az ? 1 : 0, zhi = az ? s.nz - 1 : 1;
  if (zlo < s.zown0) zlo = s.zown0;
  if (zhi > s.zown1) zhi = s.zown1;
  const bool inxy = (ay ? (gy >= 1 && gy < s.ny - 1) : gy == 0) && (ax ? (gx >= 1 && gx < s.nx - 1) : gx == 0);
  int64_t zb = zlo + (int64_t)blockIdx.z * zchunk, ze = zb + zchunk;
  if (ze > zhi) ze = zhi;

  double acc[kDerivSlots];
#pragma unroll
  for (int k = 0; k < kDerivSlots; k++) acc[k] = op_identity(deriv_op(k));

  const bool own = gx < s.nx && gy < s.ny;
  const int64_t col = gy * s.nx + gx;
  double xm = 0, x0 = 0, xp = 0, ym = 0, y0 = 0, yp = 0;
  if (own && zb < ze) {
    x0 = s.xp(zb)[col]; y0 = s.yp(zb)[col];
    if (az) { xm = s.xp(zb - 1)[col]; ym = s.yp(zb - 1)[col]; }
  }
  for (int64_t z = zb; z < ze; z++) {
    if (own && az) { xp = s.xp(z + 1)[col]; yp = s.yp(z + 1)[col]; }
    const float* Xz = s.xp(z);
    const float* Yz = s.yp(z);
    // stage plane z (own + 1-cell halo) as doubles
    for (int i = tid; i < (kTY + 2) * (kTX + 2); i += kTX * kTY) {
      const int r = i / (kTX + 2), c = i % (kTX + 2);
      const int64_t yy = (int64_t)blockIdx.y * kTY + r - 1, xx = (int64_t)blockIdx.x * kTX + c - 1;
      double vx = 0, vy = 0;
      if (yy >= 0 && yy < s.ny && xx >= 0 && xx < s.nx) {
        vx = Xz[yy * s.nx + xx];
        vy = Yz[yy * s.nx + xx];
      }
      sx[r][c] = vx;
      sy[r][c] = vy;
    }
    __syncthreads();
    if (own && inxy) {
      double Fx[CZC_NDERIV], Fy[CZC_NDERIV];
      deriv_fields(x0, xp, xm, sx[ty + 2][tx + 1], sx[ty][tx + 1], sx[ty + 1][tx + 2], sx[ty + 1][tx], az, ay, ax, Fx);
      deriv_fields(y0, yp, ym, sy[ty + 2][tx + 1], sy[ty][tx + 1], sy[ty + 1][tx + 2], sy[ty + 1][tx], az, ay, ax, Fy);
#pragma unroll
      for (int f = 0; f < CZC_NDERIV; f++) {
        const double d = Fy[f] - Fx[f];
        double* a = acc + f * kDerivStats;
        a[0] = fmax(a[0], fabs(d));
        a[1] += fabs(d);
        a[2] = fma(d, d, a[2]);
        a[3] = fmin(a[3], Fx[f]);
        a[4] = fmax(a[4], Fx[f]);
      }
    }
    __syncthreads();
    xm = x0; x0 = xp; ym = y0; y0 = yp;
  }

  const unsigned bid = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
  block_reduce_slots<kDerivSlots>(acc, DerivOp{}, parts + (size_t)bid * kDerivSlots);
  if (!last_block_arrive(ticket)) return;
  finish_slots<kDerivSlots>(parts, gridDim.x * gridDim.y * gridDim.z, DerivOp{}, res->deriv);
  if (tid == 0) *ticket = 0;
}

// ------------------------------------------------------------------------------------------------
// Autocorrelation (Eq. 2).  Ring of T+1 planes of eps = e - mu (FP64) in shared memory, tile of
// 32 x 8 points plus a +T halo in x and y.  Point p of plane zp is processed once planes
// zp..zp+T are resident; lag tau contributes iff p in R_tau, i.e. tau <= m(p) = min over active
// axes of (n_a - 1 - p_a).  S(tau) accumulates eps_p * sum_a eps_{p + tau e_a}.
// ------------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(kTX * kTY)
ac_kernel(Field3 s, int T, int zchunk,
          double* __restrict__ parts, DevResults* __restrict__ res, unsigned int* __restrict__ ticket) {
  extern __shared__ double ring[];   // [(T+1)][kTY+T][kTX+T]
  const int tx = threadIdx.x, ty = threadIdx.y, tid = ty * kTX + tx;
  const int FY = kTY + T, FX = kTX + T, R = T + 1;
  const int64_t gx = (int64_t)blockIdx.x * kTX + tx, gy = (int64_t)blockIdx.y * kTY + ty;
  const bool az = s.nz > 1, ay = s.ny > 1, ax = s.nx > 1;
  const int64_t plane = s.ny * s.nx;
  const double mu = res->p1.me;
  const int64_t zb = s.zown0 + (int64_t)blockIdx.z * zchunk;
  int64_t ze = zb + zchunk;
  if (ze > s.zown1) ze = s.zown1;

  double acc[kAcSlots];
#pragma unroll
  for (int k = 0; k < kAcSlots; k++) acc[k] = 0;

  auto load_plane = [&](int64_t zl) {
    double* dst = ring + (size_t)(zl % R) * FY * FX;
    const float* Xz = s.xp(zl);
    const float* Yz = s.yp(zl);
    for (int i = tid; i < FY * FX; i += kTX * kTY) {
      const int r = i / FX, c = i % FX;
      const int64_t yy = (int64_t)blockIdx.y * kTY + r, xx = (int64_t)blockIdx.x * kTX + c;
      double v = 0;
      if (yy < s.ny && xx < s.nx) {
        const int64_t idx = yy * s.nx + xx;
        v = ((double)Yz[idx] - (double)Xz[idx]) - mu;
      }
      dst[i] = v;
    }
  };
  // m(p) over the in-plane axes (z handled per plane)
  int64_t mxy = INT64_MAX;
  if (ay) mxy = min(mxy, s.ny - 1 - gy);
  if (ax) mxy = min(mxy, s.nx - 1 - gx);
  const bool own = gx < s.nx && gy < s.ny;

  if (zb < ze) {
    const int64_t pre_end = (zb + (int64_t)T < s.nz) ? zb + (int64_t)T : s.nz;   // planes zb .. zb+T-1
    for (int64_t zl = zb; zl < pre_end; zl++) load_plane(zl);
  }
  for (int64_t zp = zb; zp < ze; zp++) {
    if (zp + T < s.nz) load_plane(zp + T);
    __syncthreads();
    if (own) {
      int64_t m = mxy;
      if (az) m = min(m, s.nz - 1 - zp);
      const int mlim = (int)(m < (int64_t)T ? m : (int64_t)T);
      const int sp = (int)(zp % R);
      const double* P0 = ring + (size_t)sp * FY * FX;
      const double ep = P0[ty * FX + tx];
#pragma unroll
      for (int tau = 1; tau <= CZC_MAX_LAG; tau++) {
        if (tau <= mlim) {
          double nb = 0;
          if (az) {
            int sl = sp + tau;
            if (sl >= R) sl -= R;
            nb += ring[(size_t)sl * FY * FX + ty * FX + tx];
          }
          if (ay) nb += P0[(ty + tau) * FX + tx];
          if (ax) nb += P0[ty * FX + tx + tau];
          acc[tau - 1] = fma(ep, nb, acc[tau - 1]);
        }
      }
    }
    __syncthreads();
  }

  const unsigned bid = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
  block_reduce_slots<kAcSlots>(acc, SumOp{}, parts + (size_t)bid * kAcSlots);
  if (!last_block_arrive(ticket)) return;
  finish_slots<kAcSlots>(parts, gridDim.x * gridDim.y * gridDim.z, SumOp{}, res->ac);
  if (tid == 0) *ticket = 0;
}

static inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

static int64_t deriv_zplanes(const Field3& s) {
  int64_t zlo = s.nz > 1 ? 1 : 0, zhi = s.nz > 1 ? s.nz - 1 : 1;
  if (zlo < s.zown0) zlo = s.zown0;
  if (zhi > s.zown1) zhi = s.zown1;
  return zhi > zlo ? zhi - zlo : 1;
}
int64_t deriv_blocks(const Field3& s, int zchunk) {
  return cdiv(s.nx, kTX) * cdiv(s.ny, kTY) * cdiv(deriv_zplanes(s), zchunk);
}
int64_t ac_blocks(const Field3& s, int zchunk) {
  const int64_t nzo = s.zown1 > s.zown0 ? s.zown1 - s.zown0 : 1;
  return cdiv(s.nx, kTX) * cdiv(s.ny, kTY) * cdiv(nzo, zchunk);
}
size_t ac_smem_bytes(int T) { return (size_t)(T + 1) * (kTY + T) * (kTX + T) * sizeof(double); }

cudaError_t launch_deriv(const Field3& s, int zchunk, double* parts, DevResults* res,
                         unsigned int* ticket, cudaStream_t st) {
  dim3 grid((unsigned)cdiv(s.nx, kTX), (unsigned)cdiv(s.ny, kTY), (unsigned)cdiv(deriv_zplanes(s), zchunk));
  deriv_kernel<<<grid, dim3(kTX, kTY), 0, st>>>(s, zchunk, parts, res, ticket);
  return cudaGetLastError();
}

cudaError_t launch_ac(const Field3& s, int T, int zchunk, double* parts, DevResults* res,
                      unsigned int* ticket, cudaStream_t st) {
  const size_t smem = ac_smem_bytes(T);
  cudaError_t e = cudaFuncSetAttribute(ac_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  const int64_t nzo = s.zown1 > s.zown0 ? s.zown1 - s.zown0 : 1;
  dim3 grid((unsigned)cdiv(s.nx, kTX), (unsigned)cdiv(s.ny, kTY), (unsigned)cdiv(nzo, zchunk));
  ac_kernel<<<grid, dim3(kTX, kTY), smem, st>>>(s, T, zchunk, parts, res, ticket);
  return cudaGetLastError();
}

}  // namespace czc

// Second pipe probe (design input for the SSIM / AC / derivative rewrites): throughput of the
// instructions the kernels are made of, each with 8 independent chains per thread at full
// occupancy, and mixes that show whether two instruction kinds share a pipe.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/probe/pipes2 tools/probe/pipes2.cu
#include <cstdio>
#include <cuda_runtime.h>
#define ITERS 2048

__device__ __forceinline__ double cvt_fd(float f) { double d; asm volatile("cvt.f64.f32 %0, %1;" : "=d"(d) : "f"(f)); return d; }
__device__ __forceinline__ float cvt_df(double d) { float f; asm volatile("cvt.rn.f32.f64 %0, %1;" : "=f"(f) : "d"(d)); return f; }
__device__ __forceinline__ double dfma(double a, double b, double c) { double d; asm volatile("fma.rn.f64 %0, %1, %2, %3;" : "=d"(d) : "d"(a), "d"(b), "d"(c)); return d; }
__device__ __forceinline__ unsigned lop(unsigned a, unsigned b) { unsigned d; asm volatile("xor.b32 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b)); return d; }
__device__ __forceinline__ unsigned shr(unsigned a) { unsigned d; asm volatile("shr.u32 %0, %1, 3;" : "=r"(d) : "r"(a)); return d; }
__device__ __forceinline__ unsigned iadd(unsigned a, unsigned b) { unsigned d; asm volatile("add.u32 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b)); return d; }
__device__ __forceinline__ float ffma(float a, float b, float c) { float d; asm volatile("fma.rn.f32 %0, %1, %2, %3;" : "=f"(d) : "f"(a), "f"(b), "f"(c)); return d; }
__device__ __forceinline__ float fmn(float a, float b) { float d; asm volatile("min.f32 %0, %1, %2;" : "=f"(d) : "f"(a), "f"(b)); return d; }
__device__ __forceinline__ double rcp64(double a) { double d; asm volatile("rcp.approx.ftz.f64 %0, %1;" : "=d"(d) : "d"(a)); return d; }
__device__ __forceinline__ float shfl(float v, int o) { float d; asm volatile("shfl.sync.down.b32 %0, %1, %2, 0x1f, 0xffffffff;" : "=f"(d) : "f"(v), "r"(o)); return d; }
__device__ __forceinline__ double dmin(double a, double b) { double d; asm volatile("min.f64 %0, %1, %2;" : "=d"(d) : "d"(a), "d"(b)); return d; }
// float -> double by integer bit placement (exact for every finite float incl. 0 / subnormals):
// the result is x * 2^-896; callers fold 2^896 into a DFMA.
__device__ __forceinline__ double bits_fd(float f) {
  const unsigned u = __float_as_uint(f);
  const unsigned hi = (unsigned)(((int)u) >> 3) & 0x8FFFFFFFu, lo = u << 29;
  return __hiloint2double((int)hi, (int)lo);
}

template <int OP>
__global__ void k(double* dout, float* fout, unsigned* uout, float a, double b) {
  double d[8]; float f[8]; unsigned u[8];
#pragma unroll
  for (int i = 0; i < 8; i++) { d[i] = threadIdx.x * 1e-3 + i; f[i] = threadIdx.x * 1e-3f + i; u[i] = threadIdx.x * 7 + i; }
  const unsigned ku = __float_as_uint(a);
  for (int it = 0; it < ITERS; it++) {
#pragma unroll
    for (int i = 0; i < 8; i++) {
      if (OP == 0) d[i] = dfma(d[i], b, b);                                   // DFMA
      if (OP == 1) { d[i] = cvt_fd(f[i]); f[i] = __uint_as_float(lop(__float_as_uint(f[i]), __double2hiint(d[i]))); }  // F2F.F64.F32 + LOP
      if (OP == 2) u[i] = lop(u[i], ku);                                      // LOP3
      if (OP == 3) { d[i] = dfma(d[i], b, b); if (i < 2) d[i] = dfma(cvt_fd(f[i]), b, d[i]); }  // 8 DFMA + 2 F2F (shares?)
      if (OP == 4) { d[i] = dfma(bits_fd(f[i]), b, d[i]); f[i] = __uint_as_float(iadd(__float_as_uint(f[i]), ku)); }  // int-trick conv + DFMA
      if (OP == 5) f[i] = shfl(f[i], i + 1);                                  // SHFL
      if (OP == 6) f[i] = ffma(f[i], a, a);                                   // FFMA
      if (OP == 7) f[i] = fmn(f[i], a + i);                                   // FMNMX
      if (OP == 8) u[i] = shr(u[i]) + ku;                                     // SHF + IADD
      if (OP == 9) { f[i] = cvt_df(d[i]); d[i] = __hiloint2double(__float_as_int(f[i]), 0); }   // F2F.F32.F64
      if (OP == 10) d[i] = rcp64(d[i]);                                       // MUFU.RCP64H
      if (OP == 11) d[i] = dmin(d[i], b + i);                                 // DMNMX
      if (OP == 12) { d[i] = dfma(d[i], b, b); f[i] = ffma(f[i], a, a); }     // DFMA + FFMA co-issue
      if (OP == 13) { d[i] = dfma(d[i], b, b); u[i] = lop(u[i], ku); }        // DFMA + LOP co-issue
      if (OP == 14) { f[i] = ffma(f[i], a, a); u[i] = lop(u[i], ku); }        // FFMA + LOP co-issue
      if (OP == 15) { d[i] = dfma(d[i], b, b); if (i < 2) d[i] = dmin(d[i], b); }  // DFMA + DMNMX (shares?)
    }
  }
  double sd = 0; float sf = 0; unsigned su = 0;
#pragma unroll
  for (int i = 0; i < 8; i++) { sd += d[i]; sf += f[i]; su ^= u[i]; }
  const int g = blockIdx.x * blockDim.x + threadIdx.x;
  dout[g] = sd; fout[g] = sf; uout[g] = su;
}

__global__ void lds128(double* out) {
  __shared__ double2 s[2048];
  for (int i = threadIdx.x; i < 2048; i += blockDim.x) s[i] = make_double2(i, i);
  __syncthreads();
  double2 acc[4] = {};
  const int idx = threadIdx.x;
  for (int it = 0; it < ITERS; it++) {
#pragma unroll
    for (int j = 0; j < 4; j++) { const double2 v = s[(idx + it * 4 + j * 512) & 2047]; acc[j].x += v.x; acc[j].y += v.y; }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc[0].x + acc[1].y + acc[2].x + acc[3].y;
}

static int g_sms, g_clk;
template <int OP>
void run(const char* name, double ops_per_inner) {
  const int blocks = g_sms * 8, threads = 256;
  double* dout; float* fout; unsigned* uout;
  cudaMalloc(&dout, blocks * threads * 8); cudaMalloc(&fout, blocks * threads * 4); cudaMalloc(&uout, blocks * threads * 4);
  k<OP><<<blocks, threads>>>(dout, fout, uout, 1.0001f, 0.9999);
  cudaDeviceSynchronize();
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  float best = 1e9;
  for (int r = 0; r < 3; r++) {
    cudaEventRecord(e0); k<OP><<<blocks, threads>>>(dout, fout, uout, 1.0001f, 0.9999); cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
  }
  const double n = (double)blocks * threads * ITERS * 8 * ops_per_inner;
  printf("%-44s %8.3f ms  %7.1f thread-ops/clk/SM\n", name, best, n / (best * 1e-3) / g_sms / (g_clk * 1e3));
  cudaFree(dout); cudaFree(fout); cudaFree(uout);
}

int main() {
  cudaDeviceGetAttribute(&g_sms, cudaDevAttrMultiProcessorCount, 0);
  cudaDeviceGetAttribute(&g_clk, cudaDevAttrClockRate, 0);
  printf("SMs %d, clock %d MHz; rates are per inner op (counted as noted)\n", g_sms, g_clk / 1000);
  run<0>("DFMA", 1);
  run<1>("F2F.F64.F32 (+LOP3) [per F2F]", 1);
  run<2>("LOP3", 1);
  run<3>("DFMA x8 + F2F x2 [per DFMA]", 1);
  run<4>("int conv (SHF,LOP3,SHL)+DFMA+IADD [per elem]", 1);
  run<5>("SHFL.DOWN (32-bit)", 1);
  run<6>("FFMA", 1);
  run<7>("FMNMX", 1);
  run<8>("SHF + IADD [per pair]", 1);
  run<9>("F2F.F32.F64 (+MOV) [per F2F]", 1);
  run<10>("MUFU.RCP64H", 1);
  run<11>("DMNMX", 1);
  run<12>("DFMA + FFMA [per pair]", 1);
  run<13>("DFMA + LOP3 [per pair]", 1);
  run<14>("FFMA + LOP3 [per pair]", 1);
  run<15>("DFMA x8 + DMNMX x2 [per DFMA]", 1);
  {
    double* out; cudaMalloc(&out, g_sms * 8 * 512 * 8);
    lds128<<<g_sms * 8, 256>>>(out); cudaDeviceSynchronize();
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0); lds128<<<g_sms * 8, 256>>>(out); cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    const double bytes = (double)g_sms * 8 * 256 * ITERS * 4 * 16;
    printf("LDS.128: %.3f ms  %.1f B/clk/SM\n", ms, bytes / (ms * 1e-3) / g_sms / (g_clk * 1e3));
  }
  return 0;
}

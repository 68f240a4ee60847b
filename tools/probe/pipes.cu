// Micro-probe of per-SM instruction throughput on B200 (design input for the SSIM / P2 kernels).
#include <cstdio>
#include <cuda_runtime.h>
#define ITERS 4096
template<int OP> __global__ void k(float* fo, double* dout, float a, double b) {
  float f0 = threadIdx.x * 1e-3f + a, f1 = f0 + 1, f2 = f0 + 2, f3 = f0 + 3;
  double d0 = threadIdx.x * 1e-3 + b, d1 = d0 + 1, d2 = d0 + 2, d3 = d0 + 3;
  #pragma unroll 16
  for (int i = 0; i < ITERS; i++) {
    if (OP == 0) { d0 = d0 + b; d1 = d1 + b; d2 = d2 + b; d3 = d3 + b; }            // DADD
    if (OP == 1) { d0 = fma(d0, b, b); d1 = fma(d1, b, b); d2 = fma(d2, b, b); d3 = fma(d3, b, b); } // DFMA
    if (OP == 2) { d0 += (double)f0; d1 += (double)f1; f0 += a; f1 += a; }           // F2F + DADD + FADD
    if (OP == 3) { f0 = fmaxf(f0, a); f1 = fminf(f1, a); f2 = fmaxf(f2, f1); f3 = fminf(f3, f0); } // FMNMX
    if (OP == 4) { f0 = fmaf(f0, a, f1); f1 = fmaf(f1, a, f2); f2 = fmaf(f2, a, f3); f3 = fmaf(f3, a, f0); } // FFMA
    if (OP == 5) { d0 = fmax(d0, b); d1 = fmin(d1, b); d2 = fmax(d2, d1); d3 = fmin(d3, d0); } // DMNMX
    if (OP == 6) { f0 = (float)d0; d0 = (double)f0 * b; }                              // F2F both ways + DMUL
  }
  fo[blockIdx.x * blockDim.x + threadIdx.x] = f0 + f1 + f2 + f3;
  dout[blockIdx.x * blockDim.x + threadIdx.x] = d0 + d1 + d2 + d3;
}
__global__ void lds(double* out, int n) {
  __shared__ double s[2048];
  for (int i = threadIdx.x; i < 2048; i += blockDim.x) s[i] = i;
  __syncthreads();
  double acc = 0; int idx = threadIdx.x;
  #pragma unroll 16
  for (int i = 0; i < ITERS; i++) { acc += s[(idx + i) & 2047]; }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
template<int OP> void run(const char* name, int opsPerIter) {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int blocks = sms * 4, threads = 512;
  float* fo; double* dout; cudaMalloc(&fo, blocks*threads*4); cudaMalloc(&dout, blocks*threads*8);
  k<OP><<<blocks, threads>>>(fo, dout, 1.0001f, 0.9999); cudaDeviceSynchronize();
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0); k<OP><<<blocks, threads>>>(fo, dout, 1.0001f, 0.9999); cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  double ops = (double)blocks*threads*ITERS*opsPerIter;
  printf("%-28s %8.3f ms  %8.1f Gop/s  %6.1f thread-ops/clk/SM (at %d MHz nominal)\n", name, ms, ops/ms/1e6, ops/(ms*1e-3)/sms/(clk*1e3), clk/1000);
  cudaFree(fo); cudaFree(dout);
}
int main() {
  run<0>("DADD", 4); run<1>("DFMA", 4); run<2>("F2F.F64.F32 (+DADD,FADD)", 2); run<3>("FMNMX", 4);
  run<4>("FFMA (3reg)", 4); run<5>("DMNMX(fmin double)", 4); run<6>("F2F both ways + DMUL", 1);
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double* out; cudaMalloc(&out, sms*4*512*8);
  lds<<<sms*4, 512>>>(out, 0); cudaDeviceSynchronize();
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0); lds<<<sms*4, 512>>>(out, 0); cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  double ops = (double)sms*4*512*ITERS;
  printf("LDS.64 %8.3f ms  %6.1f lane-loads/clk/SM\n", ms, ops/(ms*1e-3)/sms/(clk*1e3));
  return 0;
}

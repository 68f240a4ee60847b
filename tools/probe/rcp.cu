// Probe: relative error of rcp.approx.ftz.f64 alone and after one / two Newton steps.
#include <cstdio>
#include <cstdint>
#include <cmath>
__global__ void k(double* out, int n) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  uint64_t h = (uint64_t)i * 0x9E3779B97F4A7C15ull; h ^= h >> 29; h *= 0xBF58476D1CE4E5B9ull; h ^= h >> 32;
  // random float in a wide range
  float f = __uint_as_float((unsigned)(0x30800000u + (h % 0x1E000000u)));   // ~2^-30 .. 2^30
  double v = f;
  double r0; asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r0) : "d"(v));
  double e = fma(-v, r0, 1.0); double r1 = fma(r0, e, r0);
  e = fma(-v, r1, 1.0); double r2 = fma(r1, e, r1);
  double t = 1.0 / v;
  out[3 * i] = fabs(r0 - t) / t; out[3 * i + 1] = fabs(r1 - t) / t; out[3 * i + 2] = fabs(r2 - t) / t;
}
int main() {
  const int n = 1 << 22; double* d; cudaMalloc(&d, 3 * n * sizeof(double));
  k<<<n / 256, 256>>>(d, n);
  double* h = new double[3 * n]; cudaMemcpy(h, d, 3 * n * sizeof(double), cudaMemcpyDeviceToHost);
  double m[3] = {0, 0, 0};
  for (int i = 0; i < n; i++) for (int j = 0; j < 3; j++) m[j] = fmax(m[j], h[3 * i + j]);
  printf("max rel err: approx %.3e  1 newton %.3e  2 newton %.3e\n", m[0], m[1], m[2]);
}

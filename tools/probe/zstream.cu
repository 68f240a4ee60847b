// Bandwidth probe for the access patterns of the z-streaming kernels (design input):
//   flat   — grid-stride float4 stream over both arrays (P1's pattern)
//   zwalkK — thread <-> K consecutive columns of a 100 x 500 x 500 pair, walking all planes
//            (the derivative / AC / SSIM pattern: per warp 128*K B per plane per array)
//   zwalkKc— same, z split into 2 chunks (more blocks)
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/probe/zstream tools/probe/zstream.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void flat(const float4* __restrict__ x, const float4* __restrict__ y, long n4, float* out) {
  float a = 0;
  for (long i = blockIdx.x * (long)blockDim.x + threadIdx.x; i < n4; i += (long)gridDim.x * blockDim.x) {
    const float4 u = __ldg(x + i), v = __ldg(y + i);
    a += u.x * v.y + u.z * v.w + u.y + v.x;
  }
  if (a == 12345.f) out[0] = a;
}

template <int K, int QD>
__global__ void zwalk(const float* __restrict__ x, const float* __restrict__ y, long plane, int nz, int zchunk, float* out) {
  const long c = (blockIdx.x * (long)blockDim.x + threadIdx.x) * K;
  if (c >= plane) return;
  const int z0 = blockIdx.y * zchunk, z1 = min(nz, z0 + zchunk);
  float acc = 0;
  float q[QD][2 * K];
  auto ld = [&](int z, float (&d)[2 * K]) {
    if (K == 4) {
      const float4 u = __ldg(reinterpret_cast<const float4*>(x + z * plane + c));
      const float4 v = __ldg(reinterpret_cast<const float4*>(y + z * plane + c));
      d[0] = u.x; d[1] = u.y; d[2] = u.z; d[3] = u.w; d[4] = v.x; d[5] = v.y; d[6] = v.z; d[7] = v.w;
    } else if (K == 2) {
      const float2 u = __ldg(reinterpret_cast<const float2*>(x + z * plane + c));
      const float2 v = __ldg(reinterpret_cast<const float2*>(y + z * plane + c));
      d[0] = u.x; d[1] = u.y; d[2] = v.x; d[3] = v.y;
    } else {
      d[0] = __ldg(x + z * plane + c); d[1] = __ldg(y + z * plane + c);
    }
  };
#pragma unroll
  for (int u = 0; u < QD; u++) if (z0 + u < z1) ld(z0 + u, q[u]);
  for (int z = z0; z < z1; z += QD) {
#pragma unroll
    for (int u = 0; u < QD; u++) {
      if (z + u < z1) {
#pragma unroll
        for (int k = 0; k < 2 * K; k++) acc += q[u][k] * (k + 1);
        if (z + u + QD < z1) ld(z + u + QD, q[u]);
      }
    }
  }
  if (acc == 12345.f) out[0] = acc;
}

template <typename F>
float timeit(F f) {
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  f(); cudaDeviceSynchronize();
  float best = 1e9;
  for (int r = 0; r < 5; r++) {
    cudaEventRecord(a); f(); cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b); if (ms < best) best = ms;
  }
  return best;
}

int main() {
  const int nz = 100; const long plane = 500L * 500L, n = nz * plane;
  float *x, *y, *out;
  cudaMalloc(&x, n * 4); cudaMalloc(&y, n * 4); cudaMalloc(&out, 4);
  cudaMemset(x, 0, n * 4); cudaMemset(y, 0, n * 4);
  const double bytes = 2.0 * n * 4;
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  float t = timeit([&] { flat<<<sms * 8, 256>>>((const float4*)x, (const float4*)y, n / 4, out); });
  printf("flat               %7.1f us  %6.0f GB/s\n", t * 1e3, bytes / (t * 1e-3) / 1e9);
#define RUNZ(K, QD, CH)                                                                           \
  {                                                                                               \
    dim3 g((unsigned)((plane / K + 255) / 256), (nz + CH - 1) / CH);                              \
    float t = timeit([&] { zwalk<K, QD><<<g, 256>>>(x, y, plane, nz, CH, out); });                \
    printf("zwalk K=%d QD=%2d ch=%3d %7.1f us  %6.0f GB/s  blocks %u\n", K, QD, CH, t * 1e3,       \
           bytes / (t * 1e-3) / 1e9, g.x * g.y);                                                  \
  }
  RUNZ(1, 4, 100) RUNZ(1, 8, 100) RUNZ(1, 16, 100) RUNZ(1, 8, 50) RUNZ(1, 8, 25)
  RUNZ(2, 4, 100) RUNZ(2, 8, 100) RUNZ(2, 8, 50) RUNZ(2, 8, 25)
  RUNZ(4, 4, 100) RUNZ(4, 8, 100) RUNZ(4, 8, 50) RUNZ(4, 4, 25)
  return 0;
}

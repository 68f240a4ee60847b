// TMEM ring probe: the z-window x ring of the SSIM kernel in tensor memory (4 cells x 8 slots per
// thread, 32x32b.x4 stores into slot (step mod 8), x4 load of the leaving slot, x32 load of all
// slots), fed from global memory like the kernel; checks the leaving value and the window min /
// max against the exact values at every step.  A second kernel runs concurrently on another stream.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t saddr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void st4(uint32_t a, float v0, float v1, float v2, float v3) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1, %2, %3, %4};\n\ttcgen05.wait::st.sync.aligned;"
               :: "r"(a), "r"(__float_as_uint(v0)), "r"(__float_as_uint(v1)), "r"(__float_as_uint(v2)), "r"(__float_as_uint(v3)) : "memory");
}
__device__ __forceinline__ void ld4(uint32_t a, float (&v)[4]) {
  uint32_t r0, r1, r2, r3;
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0, %1, %2, %3}, [%4];\n\ttcgen05.wait::ld.sync.aligned;"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3) : "r"(a) : "memory");
  v[0] = __uint_as_float(r0); v[1] = __uint_as_float(r1); v[2] = __uint_as_float(r2); v[3] = __uint_as_float(r3);
}
__device__ __forceinline__ void ld32(uint32_t a, float (&v)[32]) {
  uint32_t r[32];
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 {"
               "%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15, "
               "%16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];\n\t"
               "tcgen05.wait::ld.sync.aligned;"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                 "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
                 "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
                 "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
               : "r"(a) : "memory");
  for (int i = 0; i < 32; i++) v[i] = __uint_as_float(r[i]);
}
// value of cell k of thread (block, tid) at plane z
__device__ __host__ inline float val(int b, int t, int k, int z) { return (float)(((b * 7919 + t * 131 + k * 17 + z * 29) % 1000) - 500); }

__global__ void __launch_bounds__(256, 2) ring(const float* __restrict__ g, int nz, int* bad) {
  __shared__ uint32_t s_t;
  extern __shared__ unsigned char big[];
  const int warp = threadIdx.x >> 5, tid = threadIdx.x;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" :: "r"(saddr(&s_t)) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t base = s_t;
  const uint32_t ta0 = base + ((uint32_t)(32 * (warp & 3)) << 16) + (uint32_t)((warp >> 2) * 128);
  int nb = 0;
  const float* gb = g + ((size_t)blockIdx.x * 256 + tid) * 4;   // [plane][block*256+tid][4]
  const size_t pstride = (size_t)gridDim.x * 256 * 4;
  float nx[4];
  for (int k = 0; k < 4; k++) nx[k] = __ldg(gb + k);
  for (int step = 0; step < nz; step++) {
    const uint32_t ta = ta0 + (uint32_t)((step & 7) * 4);
    if (step >= 8 && (step - 8) % 16 == 0) {        // "resync": planes step-7 .. step-1 by slot
      for (int t = 1; t < 8; t++) {
        float xr[4];
        ld4(ta0 + (uint32_t)(((step + t) & 7) * 4), xr);
        for (int k = 0; k < 4; k++) if (xr[k] != val(blockIdx.x, tid, k, step - 8 + t)) nb += 100;
      }
    } else if (step >= 8) {
      float xo[4];
      ld4(ta, xo);
      for (int k = 0; k < 4; k++) if (xo[k] != val(blockIdx.x, tid, k, step - 8)) nb++;
    }
    st4(ta, nx[0], nx[1], nx[2], nx[3]);
    if (step + 1 < nz) for (int k = 0; k < 4; k++) nx[k] = __ldg(gb + (size_t)(step + 1) * pstride + k);
    if (step >= 7) {
      float v[32];
      ld32(ta0, v);
      for (int k = 0; k < 4; k++) {
        float mn = v[k], mx = v[k];
        for (int t = 1; t < 8; t++) { mn = fminf(mn, v[t * 4 + k]); mx = fmaxf(mx, v[t * 4 + k]); }
        float emn = val(blockIdx.x, tid, k, step), emx = emn;
        for (int z = step - 7; z < step; z++) { emn = fminf(emn, val(blockIdx.x, tid, k, z)); emx = fmaxf(emx, val(blockIdx.x, tid, k, z)); }
        if (mn != emn || mx != emx) nb++;
      }
    }
    if ((step & 3) == 0) __syncthreads();
  }
  atomicAdd(bad, nb);
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" :: "r"(base) : "memory");
}
__global__ void noise(float* p, int n) {           // a concurrent kernel occupying warp slots
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) p[i] = p[i] * 1.0001f + 1.f;
}
int main() {
  const int blocks = 1184, nz = 40;
  const size_t n = (size_t)nz * blocks * 256 * 4;
  float* h = (float*)malloc(n * 4);
  for (int z = 0; z < nz; z++) for (int b = 0; b < blocks; b++) for (int t = 0; t < 256; t++) for (int k = 0; k < 4; k++)
    h[(((size_t)z * blocks + b) * 256 + t) * 4 + k] = val(b, t, k, z);
  float *g, *q; int* bad;
  cudaMalloc(&g, n * 4); cudaMalloc(&q, 1 << 26); cudaMalloc(&bad, 4);
  cudaMemcpy(g, h, n * 4, cudaMemcpyHostToDevice);
  cudaFuncSetAttribute(ring, cudaFuncAttributeMaxDynamicSharedMemorySize, 90000);
  cudaStream_t s1, s2; cudaStreamCreate(&s1); cudaStreamCreate(&s2);
  for (int v = 0; v < 2; v++) {
    cudaMemset(bad, 0, 4);
    if (v) noise<<<148 * 3, 96, 0, s2>>>(q, 1 << 24);
    ring<<<blocks, 256, 88000, s1>>>(g, nz, bad);
    cudaError_t e = cudaDeviceSynchronize();
    int hb; cudaMemcpy(&hb, bad, 4, cudaMemcpyDeviceToHost);
    printf("%s: err=%s mismatches=%d\n", v ? "with concurrent kernel" : "alone", cudaGetErrorString(e), hb);
  }
  return 0;
}

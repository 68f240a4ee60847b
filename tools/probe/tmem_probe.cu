// TMEM addressing probe: each thread stores (warp, lane, col) signatures with tcgen05.st 32x32b.x4
// and reads them back; variant A puts the warp's lane quarter into address bits 31:16, variant B
// leaves them 0.  Prints mismatches per variant.
#include <cstdio>
#include <cuda_runtime.h>
#include <cstdint>
__device__ __forceinline__ uint32_t saddr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
template <bool LANEOFF>
__global__ void probe(int* bad, uint32_t* sample) {
  __shared__ uint32_t s_t;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" :: "r"(saddr(&s_t)) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t base = s_t;
  const uint32_t ta = base + (LANEOFF ? ((uint32_t)(32 * (warp & 3)) << 16) : 0u) + (uint32_t)((warp >> 2) * 128);
  for (int c = 0; c < 32; c += 4) {
    uint32_t v0 = (warp << 16) | (lane << 8) | c, v1 = v0 + 1, v2 = v0 + 2, v3 = v0 + 3;
    asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1, %2, %3, %4};\n\ttcgen05.wait::st.sync.aligned;"
                 :: "r"(ta + c), "r"(v0), "r"(v1), "r"(v2), "r"(v3) : "memory");
  }
  __syncthreads();
  int nb = 0;
  for (int c = 0; c < 32; c += 4) {
    uint32_t r0, r1, r2, r3;
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0, %1, %2, %3}, [%4];\n\ttcgen05.wait::ld.sync.aligned;"
                 : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3) : "r"(ta + c) : "memory");
    const uint32_t e = (warp << 16) | (lane << 8) | c;
    nb += (r0 != e) + (r1 != e + 1) + (r2 != e + 2) + (r3 != e + 3);
    if (blockIdx.x == 0 && c == 0) sample[threadIdx.x] = r0;
  }
  {  // the same 32 columns through one 32x32b.x32 load
    uint32_t r[32];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 {"
                 "%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15, "
                 "%16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];\n\t"
                 "tcgen05.wait::ld.sync.aligned;"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                   "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
                   "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
                   "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
                 : "r"(ta) : "memory");
    for (int i = 0; i < 32; i++) {
      const uint32_t e = ((warp << 16) | (lane << 8) | (i & ~3)) + (i & 3);
      if (r[i] != e) { nb += 1000; if (blockIdx.x == 0 && lane == 0 && warp == 0) printf("x32 col %d: got %08x want %08x\n", i, r[i], e); }
    }
  }
  atomicAdd(bad, nb);
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" :: "r"(base) : "memory");
}
int main() {
  int* bad; uint32_t* smp; cudaMalloc(&bad, 4); cudaMalloc(&smp, 256 * 4);
  uint32_t h[256];
  for (int v = 0; v < 2; v++) {
    cudaMemset(bad, 0, 4);
    if (v == 0) probe<true><<<296, 256>>>(bad, smp); else probe<false><<<296, 256>>>(bad, smp);
    cudaError_t e = cudaDeviceSynchronize();
    int hb = -1; cudaMemcpy(&hb, bad, 4, cudaMemcpyDeviceToHost); cudaMemcpy(h, smp, sizeof(h), cudaMemcpyDeviceToHost);
    printf("variant %s: err=%s mismatches=%d  sample w0l0=%08x w1l0=%08x w4l0=%08x w5l3=%08x\n", v == 0 ? "A(lane offset)" : "B(no offset)",
           cudaGetErrorString(e), hb, h[0], h[32], h[128], h[163]);
    if (e != cudaSuccess) return 1;
  }
  return 0;
}

// Microbenchmark (dev tool): tcgen05.ld / tcgen05.st throughput per SM.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ inline uint32_t sa(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int NW, bool WAIT_EACH>
__global__ void k(unsigned long long *out, float *sink, int iters) {
  __shared__ uint32_t slot;
  const int tid = threadIdx.x, warp = tid >> 5;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(sa(&slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tl = slot + ((uint32_t)((warp & 3) * 32) << 16) + (uint32_t)((warp >> 2) * 256);
  float acc = 0.f;
  __syncthreads();
  unsigned long long t0 = clock64();
  for (int i = 0; i < iters; ++i) {
    uint32_t r[16];
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
        : "r"(tl + (uint32_t)((i & 7) * 16)));
    if (WAIT_EACH || (i & 3) == 3) asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
    for (int j = 0; j < 16; ++j) acc += __uint_as_float(r[j]);
  }
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
  __syncthreads();
  unsigned long long t1 = clock64();
  if (tid == 0 && blockIdx.x == 0) out[0] = t1 - t0;
  sink[blockIdx.x * blockDim.x + tid] = acc;
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(slot));
}

template <int NW, bool W>
void run() {
  unsigned long long *d, h = 0;
  float *sink;
  cudaMalloc(&d, 8);
  cudaMalloc(&sink, 148 * 1024 * 4);
  const int iters = 4096;
  k<NW, W><<<148, NW * 32>>>(d, sink, iters);
  k<NW, W><<<148, NW * 32>>>(d, sink, iters);
  cudaError_t e = cudaDeviceSynchronize();
  cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
  const double bytes = (double)NW * iters * 32 * 16 * 4;
  printf("warps %d wait_each %d: %s  %.1f bytes/cycle/SM (%.0f cycles)\n", NW, (int)W, cudaGetErrorString(e),
         bytes / h, (double)h);
}

int main() {
  run<4, true>();
  run<4, false>();
  run<8, true>();
  run<8, false>();
  return 0;
}

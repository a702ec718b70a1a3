// Microbenchmark (dev tool): cycles per tcgen05.mma kind::tf32 issued back to
// back by one thread, for a few N and smem-descriptor layouts.  Operand data
// is garbage; only the issue/execute rate is measured.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ inline uint32_t sa(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int N, int LAYOUT>
__global__ void k(unsigned long long *out, int iters) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ uint32_t slot;
  __shared__ __align__(8) uint64_t bar;
  const int tid = threadIdx.x;
  if (tid < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(sa(&slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = slot;
  const uint32_t base = sa(sm);
  // SWIZZLE_NONE: LBO 128 B, SBO 256 B; SWIZZLE_128B (layout 2): LBO 16 B (ignored), SBO 1024 B
  const uint64_t lbo = LAYOUT == 0 ? (128 >> 4) : 1, sbo = LAYOUT == 0 ? (256 >> 4) : (1024 >> 4);
  const uint64_t da = ((uint64_t)((base & 0x3FFFF) >> 4)) | (lbo << 16) | (sbo << 32) | (1ull << 46) |
                      ((uint64_t)(LAYOUT == 0 ? 0 : 2) << 61);
  const uint64_t db = ((uint64_t)(((base + 65536) & 0x3FFFF) >> 4)) | (lbo << 16) | (sbo << 32) | (1ull << 46) |
                      ((uint64_t)(LAYOUT == 0 ? 0 : 2) << 61);
  const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
  if (tid == 0) {
    unsigned long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n"
                   ::"r"(tmem), "l"(da), "l"(db), "r"(idesc), "r"(i));
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(sa(&bar)) : "memory");
    asm volatile("{\n.reg .pred P1;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n@!P1 bra W;\n}\n" ::"r"(sa(&bar)) : "memory");
    unsigned long long t1 = clock64();
    if (blockIdx.x == 0) out[0] = t1 - t0;
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (tid < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" ::"r"(tmem));
}

template <int N, int LAYOUT>
void run(const char *name) {
  unsigned long long *d, h = 0;
  cudaMalloc(&d, 8);
  const int smem = 160 * 1024;
  cudaFuncSetAttribute(k<N, LAYOUT>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int iters = 4096;
  k<N, LAYOUT><<<148, 128, smem>>>(d, iters);
  k<N, LAYOUT><<<148, 128, smem>>>(d, iters);
  cudaError_t e = cudaDeviceSynchronize();
  cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
  printf("%-28s N=%3d: %s  %.1f cycles per MMA (M128 K8 tf32)\n", name, N, cudaGetErrorString(e), (double)h / iters);
  cudaFree(d);
}

int main() {
  run<64, 0>("swizzle none");
  run<128, 0>("swizzle none");
  run<256, 0>("swizzle none");
  run<64, 2>("swizzle 128B");
  run<128, 2>("swizzle 128B");
  run<256, 2>("swizzle 128B");
  return 0;
}

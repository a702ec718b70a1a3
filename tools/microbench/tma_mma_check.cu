// Dev check: TMA (4-D tensor map, SWIZZLE_128B, fp32 box 32 x 128) feeding
// tcgen05.mma kind::tf32 with SWIZZLE_128B K-major smem descriptors.
// D[128][64] = A[128][64] . B[64][64]^T (B stored [n][k], k contiguous).
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cmath>
#include <vector>
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

__device__ inline uint32_t sa(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ inline uint64_t desc_sw128(uint32_t saddr) {
  return (uint64_t)((saddr & 0x3FFFF) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}

__global__ void k(const __grid_constant__ CUtensorMap ta, const __grid_constant__ CUtensorMap tb, float *out) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ __align__(8) uint64_t bar, mbar;
  __shared__ uint32_t slot;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  unsigned char *A = sm;              // 2 x 16 KB (k 0-31, k 32-63)
  unsigned char *B = sm + 32768;      // 2 x 8 KB
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 64;" ::"r"(sa(&slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&bar)));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&mbar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = slot;
  if (tid == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(&bar)), "r"(49152) : "memory");
    for (int h = 0; h < 2; ++h) {
      // A: coords {x=32h, row=0, c=0, buf=0}
      asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];"
                   ::"r"(sa(A + h * 16384)), "l"(&ta), "r"(32 * h), "r"(0), "r"(0), "r"(0), "r"(sa(&bar)) : "memory");
      asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];"
                   ::"r"(sa(B + h * 8192)), "l"(&tb), "r"(32 * h), "r"(0), "r"(0), "r"(0), "r"(sa(&bar)) : "memory");
    }
    asm volatile("{\n.reg .pred P1;\nW1:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n@!P1 bra W1;\n}\n" ::"r"(sa(&bar)) : "memory");
    const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(64 >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    for (int kk = 0; kk < 8; ++kk) {
      const int h = kk >> 2, kin = kk & 3;
      const uint64_t da = desc_sw128(sa(A + h * 16384) + kin * 32);
      const uint64_t db = desc_sw128(sa(B + h * 8192) + kin * 32);
      asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n"
                   ::"r"(tmem), "l"(da), "l"(db), "r"(idesc), "r"(kk));
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(sa(&mbar)) : "memory");
  }
  __syncwarp();
  asm volatile("{\n.reg .pred P1;\nW2:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n@!P1 bra W2;\n}\n" ::"r"(sa(&mbar)) : "memory");
  asm volatile("tcgen05.fence::after_thread_sync;");
  if (warp < 4) {
    for (int q = 0; q < 4; ++q) {
      uint32_t r[16];
      asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                   : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                     "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                   : "r"(tmem + ((uint32_t)(warp * 32) << 16) + q * 16));
      asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
      for (int i = 0; i < 16; ++i) out[(warp * 32 + lane) * 64 + q * 16 + i] = __uint_as_float(r[i]);
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 64;" ::"r"(tmem));
}

static float tf32t(float x) { uint32_t b; memcpy(&b, &x, 4); b &= 0xffffe000u; memcpy(&x, &b, 4); return x; }

int main() {
  PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void **)&enc, cudaEnableDefault, &q);
  if (!enc) { printf("no cuTensorMapEncodeTiled\n"); return 1; }
  const int P = 256, S = 64;   // A global [buf=1][c=1][P][64], tile at row 0
  std::vector<float> hA(P * S), hB(S * S);
  srand(1);
  for (auto &v : hA) v = (float)rand() / RAND_MAX;
  for (auto &v : hB) v = (float)rand() / RAND_MAX;
  float *dA, *dB, *dO;
  cudaMalloc(&dA, hA.size() * 4); cudaMalloc(&dB, hB.size() * 4); cudaMalloc(&dO, 128 * 64 * 4);
  cudaMemcpy(dA, hA.data(), hA.size() * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(dB, hB.data(), hB.size() * 4, cudaMemcpyHostToDevice);
  CUtensorMap ta, tb;
  cuuint64_t gdA[4] = {64, (cuuint64_t)P, 1, 1}, gsA[3] = {256, (cuuint64_t)P * 256, (cuuint64_t)P * 256};
  cuuint32_t box[4] = {32, 128, 1, 1}, es[4] = {1, 1, 1, 1};
  CUresult r1 = enc(&ta, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, dA, gdA, gsA, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                    CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  cuuint64_t gdB[4] = {64, 64, 1, 1}, gsB[3] = {256, 64 * 256, 64 * 256};
  cuuint32_t boxB[4] = {32, 64, 1, 1};
  CUresult r2 = enc(&tb, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, dB, gdB, gsB, boxB, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                    CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  printf("encode %d %d\n", (int)r1, (int)r2);
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 49152 + 1024);
  k<<<1, 128, 49152 + 1024>>>(ta, tb, dO);
  cudaError_t e = cudaDeviceSynchronize();
  printf("kernel: %s\n", cudaGetErrorString(e));
  std::vector<float> hO(128 * 64);
  cudaMemcpy(hO.data(), dO, hO.size() * 4, cudaMemcpyDeviceToHost);
  double worst = 0;
  for (int i = 0; i < 128; ++i)
    for (int j = 0; j < 64; ++j) {
      double ref = 0;
      for (int kk = 0; kk < 64; ++kk) ref += (double)tf32t(hA[i * 64 + kk]) * (double)tf32t(hB[j * 64 + kk]);
      worst = fmax(worst, fabs(hO[i * 64 + j] - ref) / fabs(ref));
    }
  printf("max rel err vs tf32-truncated reference: %.3e (%s)\n", worst, worst < 1e-5 ? "OK" : "MISMATCH");
  return 0;
}

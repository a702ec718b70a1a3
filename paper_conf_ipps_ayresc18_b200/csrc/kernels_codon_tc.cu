// K3-TC: 61-state codon updatePartials on the 5th-generation tensor cores
// (tcgen05.mma kind::tf32, accumulators in TMEM), fp32 instances with c <= 4.
//
// Eq. (1) (§II-A) for s = 61 is, per operation, category c and
// 128-pattern tile, two dense products
//     D_b[p][z] = sum_x A_b[p][x] P_b[c][z][x]      (b = child 1, 2)
// followed by out = D_1 .* D_2 and the per-pattern rescale (max over (c, z)).
// This is the one place on the hot path that really is a dense contraction
// (BASELINE north star), so it runs on tcgen05:
//  * M = 128 patterns (TMEM lanes), N = 64 states (61 padded), K = 64 child
//    states in 8 steps of K = 8 (tf32).
//  * fp32 accuracy with 3xTF32: x = hi + lo with hi = x with the low 13
//    mantissa bits cleared (exact) and lo = x - hi (exact).  hi*hi goes to a
//    main accumulator, hi*lo + lo*hi to a separate correction accumulator: the
//    MMA aligns every addend to its accumulator's magnitude with ~20 bits, so
//    corrections ~2^-11 smaller than the main terms would lose most of their
//    bits in a shared accumulator (measured: 4e-6 vs 9e-7 per product with
//    tools/diag_codon_tc.py).  A tip child's A tile is one-hot (or all ones
//    for a missing state -> row sums), exact in tf32, so its lo*hi is skipped.
//  * TMEM: two category buffers x 2 children x (main, correction) x 64
//    columns = 512 columns, so category c+1's MMAs never wait for category
//    c's epilogue to drain TMEM.
//  * Operands are built by all 256 threads straight into the canonical
//    no-swizzle K-major UMMA layout (8-row x 16-byte core matrices; LBO = 128 B
//    between the two K halves, SBO = 256 B between 8-row groups), published to
//    the async proxy (fence.proxy.async), and one elected thread issues the
//    MMAs and tcgen05.commit's them to an mbarrier.
//  * Epilogue per category: warps 0-3 own TMEM lane quarters (one pattern per
//    thread; tcgen05.ld 32x32b.x16): (main1 + corr1) * (main2 + corr2) is
//    stored unscaled while the running max over (c, z) is kept; once all
//    categories are done the thread rescales its own rows by the exact 2^-e
//    (an L2-resident re-read of 256 B per category).
// Persistent CTAs (one per SM: the CTA owns all of TMEM) walk the flattened
// (operation, tile) space of the level set.
#include <cuda_runtime.h>

#include <cstdint>

#include "rrl_internal.h"

namespace rrl {
namespace {

constexpr int TM = 128;  // patterns per tile = MMA M = TMEM lanes
constexpr int TS = 64;   // padded states: MMA N and K
constexpr int kS61 = 61;
constexpr int kThr = 256;
constexpr int A_BYTES = TM * TS * 4;  // 32 KB per operand tile
constexpr int B_BYTES = TS * TS * 4;  // 16 KB
// smem: A[child][hi,lo], B[child][hi,lo]
constexpr int SMEM_A = 0;
constexpr int SMEM_B = 4 * A_BYTES;
constexpr int SMEM_ST = SMEM_B + 4 * B_BYTES;   // tip states [2][128]
constexpr int SMEM_BAR = SMEM_ST + 2 * TM;      // mbarrier
constexpr int SMEM_TMEM = SMEM_BAR + 8;         // TMEM base address
constexpr int SMEM_TOTAL = SMEM_TMEM + 8;

__device__ inline uint32_t smem_addr(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
// byte offset of the 16-byte chunk (row r, k-chunk j) in a K-major no-swizzle
// UMMA tile: [kb = j/2][row group r/8][k half j%2][row r%8][16 B]
__device__ inline uint32_t umma_off(int r, int j, int rows) {
  return (uint32_t)((j >> 1) * (rows * 32) + (r >> 3) * 256 + (j & 1) * 128 + (r & 7) * 16);
}
__device__ inline uint64_t umma_desc(uint32_t saddr) {
  return (uint64_t)((saddr & 0x3FFFFu) >> 4) | ((uint64_t)(128 >> 4) << 16) |
         ((uint64_t)(256 >> 4) << 32) | ((uint64_t)1 << 46);
}
// kind::tf32, D f32, A/B tf32 K-major, N = 64, M = 128
constexpr uint32_t kIdesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(TS >> 3) << 17) |
                            ((uint32_t)(TM >> 4) << 24);

__device__ inline void mma_tf32(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t acc) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n" ::"r"(tmem_d),
      "l"(a), "l"(b), "r"(kIdesc), "r"(acc));
}
__device__ inline void mma_commit(uint64_t *bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                   smem_addr(bar))
               : "memory");
}
__device__ inline void bar_wait(uint64_t *bar, uint32_t parity) {
  asm volatile(
      "{\n.reg .pred P1;\nW_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra W_%=;\n}\n" ::"r"(smem_addr(bar)),
      "r"(parity)
      : "memory");
}
__device__ inline void tmem_ld16(uint32_t taddr, float (&v)[16]) {
  uint32_t r[16];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
#pragma unroll
  for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
}
__device__ inline void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
__device__ inline void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ inline void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

__device__ inline float tf32_hi(float x) { return __uint_as_float(__float_as_uint(x) & 0xffffe000u); }

__device__ inline void sts128(uint32_t addr, float a, float b, float c, float d) {
  asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(addr), "f"(a), "f"(b), "f"(c), "f"(d)
               : "memory");
}

__device__ inline int frexp_e(float m) {
  const unsigned b = __float_as_uint(m);
  const int eb = (int)((b >> 23) & 0xffu);
  if (eb != 0 && eb != 0xff) return eb - 126;
  if (m == 0.f) return 0;
  int e;
  frexpf(m, &e);
  return e;
}

template <int C>
__global__ void __launch_bounds__(kThr, 1)
k_partials_codon_tc(const DevOp *__restrict__ ops, int p, int p_pad, int ntiles, int total) {
  extern __shared__ __align__(1024) unsigned char sm[];
  uint64_t *bar = reinterpret_cast<uint64_t *>(sm + SMEM_BAR);
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(sm + SMEM_TMEM);
  uint8_t *st_s = sm + SMEM_ST;
  const uint32_t sbase = smem_addr(sm);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;

  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_addr(tmem_slot)),
                 "r"(512));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_addr(bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *tmem_slot;

  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" :::);

  uint32_t phase = 0;
  // TMEM columns: two category buffers of 256 columns; per buffer and child b
  // the main accumulator (hi*hi) at 128 b and the correction accumulator
  // (hi*lo + lo*hi) at 128 b + 64.  Keeping the ~2^-11-smaller corrections in
  // their own accumulator keeps them accurate (the MMA aligns every addend to
  // the accumulator's magnitude with ~20 bits); they meet in fp32 in the epilogue.
  for (int f = blockIdx.x; f < total; f += gridDim.x) {
    const DevOp &op = ops[f / ntiles];
    const int p0 = (f % ntiles) * TM;
    const bool tip[2] = {(op.flags & OP_TIP1) != 0, (op.flags & OP_TIP2) != 0};
    const void *in[2] = {op.in1, op.in2};
    const float *Pg[2] = {static_cast<const float *>(op.P1), static_cast<const float *>(op.P2)};
    for (int b = 0; b < 2; ++b)
      if (tip[b] && tid < TM) {
        const int pp = p0 + tid;
        st_s[b * TM + tid] = pp < p ? static_cast<const uint8_t *>(in[b])[pp] : (uint8_t)kS61;
      }
    const int r = warp * 32 + lane;  // epilogue row (warps 0-3)
    const int pp = p0 + r;
    const bool valid = warp < 4 && pp < p;
    float *out = static_cast<float *>(op.out);
    const uint32_t lane_base = tmem + ((uint32_t)((warp & 3) * 32) << 16);
    float m = 0.f;

    // product of category cc from TMEM buffer cc&1 -> out (unscaled), running max
    auto epilogue_cat = [&](int cc) {
      const uint32_t cb = lane_base + (uint32_t)((cc & 1) * 256);
#pragma unroll
      for (int q = 0; q < TS / 16; ++q) {
        float m1[16], c1[16], m2[16], c2[16];
        tmem_ld16(cb + 0 + q * 16, m1);
        tmem_ld16(cb + 64 + q * 16, c1);
        tmem_ld16(cb + 128 + q * 16, m2);
        tmem_ld16(cb + 192 + q * 16, c2);
        tmem_wait_ld();
        float v[16];
#pragma unroll
        for (int i = 0; i < 16; ++i) {
          v[i] = (m1[i] + c1[i]) * (m2[i] + c2[i]);
          m = fmaxf(m, v[i]);
        }
        if (valid) {
          float4 *dst = reinterpret_cast<float4 *>(out + ((size_t)cc * p_pad + pp) * TS + q * 16);
#pragma unroll
          for (int i = 0; i < 4; ++i) dst[i] = make_float4(v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
        }
      }
    };

    for (int c = 0; c < C; ++c) {
      if (c > 0) {  // MMAs of category c-1 done: operand smem free, its products ready
        bar_wait(bar, phase);
        phase ^= 1u;
        fence_after();
        if (warp < 4) epilogue_cat(c - 1);
        fence_before();
      }
      __syncthreads();  // tip states visible; smem and TMEM buffer c&1 free
      // ---- operand tiles for category c (both children), hi/lo split
      for (int b = 0; b < 2; ++b) {
        const uint32_t a_hi = sbase + SMEM_A + (2 * b) * A_BYTES, a_lo = a_hi + A_BYTES;
        if (!tip[b]) {
          const float *A = static_cast<const float *>(in[b]) + ((size_t)c * p_pad + p0) * TS;
          for (int i = tid; i < TM * 16; i += kThr) {
            const int kh = i & 1, rr = (i >> 1) & (TM - 1), kb = i >> 8;
            const int j = kb * 2 + kh;
            float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
            if (p0 + rr < p) v = __ldg(reinterpret_cast<const float4 *>(A + (size_t)rr * TS + j * 4));
            const uint32_t o = umma_off(rr, j, TM);
            const float h0 = tf32_hi(v.x), h1 = tf32_hi(v.y), h2 = tf32_hi(v.z), h3 = tf32_hi(v.w);
            sts128(a_hi + o, h0, h1, h2, h3);
            sts128(a_lo + o, v.x - h0, v.y - h1, v.z - h2, v.w - h3);
          }
        } else {
          for (int i = tid; i < TM * 16; i += kThr) {
            const int kh = i & 1, rr = (i >> 1) & (TM - 1), kb = i >> 8;
            const int j = kb * 2 + kh;
            const unsigned sv = st_s[b * TM + rr];
            float v[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              const unsigned k = (unsigned)(j * 4 + q);
              v[q] = (sv < (unsigned)kS61) ? (k == sv ? 1.f : 0.f) : (k < (unsigned)kS61 ? 1.f : 0.f);
            }
            sts128(a_hi + umma_off(rr, j, TM), v[0], v[1], v[2], v[3]);
          }
        }
        const uint32_t b_hi = sbase + SMEM_B + (2 * b) * B_BYTES, b_lo = b_hi + B_BYTES;
        const float *P = Pg[b] + (size_t)c * TS * TS;  // natural [z][x] = K-major B
        for (int i = tid; i < TS * 16; i += kThr) {
          const int kh = i & 1, z = (i >> 1) & (TS - 1), kb = i >> 7;
          const int j = kb * 2 + kh;
          const float4 v = __ldg(reinterpret_cast<const float4 *>(P + z * TS + j * 4));
          const uint32_t o = umma_off(z, j, TS);
          const float h0 = tf32_hi(v.x), h1 = tf32_hi(v.y), h2 = tf32_hi(v.z), h3 = tf32_hi(v.w);
          sts128(b_hi + o, h0, h1, h2, h3);
          sts128(b_lo + o, v.x - h0, v.y - h1, v.z - h2, v.w - h3);
        }
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic writes -> async proxy
      fence_before();
      __syncthreads();
      if (tid == 0) {
        fence_after();
        for (int b = 0; b < 2; ++b) {
          const uint32_t dm = tmem + (uint32_t)((c & 1) * 256 + b * 128), dc = dm + 64;
          const uint32_t a_hi = sbase + SMEM_A + (2 * b) * A_BYTES, a_lo = a_hi + A_BYTES;
          const uint32_t b_hi = sbase + SMEM_B + (2 * b) * B_BYTES, b_lo = b_hi + B_BYTES;
#pragma unroll
          for (int kb = 0; kb < TS / 8; ++kb) {
            const uint64_t ah = umma_desc(a_hi + kb * (TM * 32)), al = umma_desc(a_lo + kb * (TM * 32));
            const uint64_t bh = umma_desc(b_hi + kb * (TS * 32)), bl = umma_desc(b_lo + kb * (TS * 32));
            mma_tf32(dm, ah, bh, kb > 0 ? 1u : 0u);
            mma_tf32(dc, ah, bl, kb > 0 ? 1u : 0u);
            if (!tip[b]) mma_tf32(dc, al, bh, 1u);
          }
        }
        mma_commit(bar);
      }
    }
    bar_wait(bar, phase);  // last category's products are in TMEM
    phase ^= 1u;
    fence_after();
    if (warp < 4) {
      epilogue_cat(C - 1);
      // ---- rescale: e from max over (c, z); rows re-read by the thread that wrote them
      int e = 0;
      if (op.scale_out != nullptr) {
        e = frexp_e(m);
        if (valid) {
          int tot = e;
          if (op.cum1 != nullptr) tot += op.cum1[pp];
          if (op.cum2 != nullptr) tot += op.cum2[pp];
          op.scale_out[pp] = tot;
        }
      } else if (op.scale_in != nullptr) {
        e = valid ? op.scale_in[pp] : 0;
      }
      if (valid && e != 0) {
        const float sc = (e > -126 && e < 126) ? __uint_as_float((unsigned)(127 - e) << 23) : ldexpf(1.f, -e);
        for (int c = 0; c < C; ++c) {
          float4 *row = reinterpret_cast<float4 *>(out + ((size_t)c * p_pad + pp) * TS);
#pragma unroll 4
          for (int i = 0; i < TS / 4; ++i) {
            float4 v = row[i];
            v.x *= sc; v.y *= sc; v.z *= sc; v.w *= sc;
            row[i] = v;
          }
        }
      }
    }
    fence_before();
    __syncthreads();  // TMEM and tip-state smem free for the next tile
    fence_after();
  }
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512));
}

template <int C>
int launch_tc(const DevOp *d_ops, int nops, int p, int p_pad, cudaStream_t st) {
  static int nsm = 0;
  if (nsm == 0) {
    cudaError_t e = cudaFuncSetAttribute(k_partials_codon_tc<C>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         SMEM_TOTAL);
    if (e != cudaSuccess) return (int)e;
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  }
  const int ntiles = (p + TM - 1) / TM;
  const long long total = (long long)ntiles * nops;
  if (total > 0x7fffffffLL) return (int)cudaErrorInvalidValue;
  const int grid = (int)(total < nsm ? total : nsm);
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kThr);
  cfg.dynamicSmemBytes = SMEM_TOTAL;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return (int)cudaLaunchKernelEx(&cfg, k_partials_codon_tc<C>, d_ops, p, p_pad, ntiles, (int)total);
}

}  // namespace

// fp32 codon instances, c in {1, 2, 4, 8}; cudaErrorNotSupported otherwise
// (the caller then uses the SIMT kernel).
int launch_update_partials_codon_tc(int c, const DevOp *d_ops, int nops, int p, int p_pad, void *stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  switch (c) {
    case 1: return launch_tc<1>(d_ops, nops, p, p_pad, st);
    case 2: return launch_tc<2>(d_ops, nops, p, p_pad, st);
    case 4: return launch_tc<4>(d_ops, nops, p, p_pad, st);
    case 8: return launch_tc<8>(d_ops, nops, p, p_pad, st);
    default: return (int)cudaErrorNotSupported;
  }
}

}  // namespace rrl
